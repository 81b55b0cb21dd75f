"""Long single-puncture evolution on the GPU: C2
(Schwarzschild m = 1, [-32, 32]^3, levels 3..8) with the extrapolating outer
boundary (R12) and with the radiative condition (R29), constraint norms
(dgr_constraints: Hamiltonian H, momentum M^i, Gamma constraint G^i) and the
lapse minimum sampled along the run.

    python tools/long_run.py [t_end=100] [samples=20]
Environment: DGR_SIGMA (KO strength, 0.4), DGR_ETA (2.0), DGR_CFL (0.25),
DGR_BC ("both" | "somm" | "extrap"), DGR_LMAX (finest level, 8),
DGR_PUNCT ("c2": offset h/4 in z as in synth.configs; "cell": at a cell centre),
DGR_UPWIND (1: lopsided advective derivatives, reading R9u), DGR_RHO (refinement
radius factor of the mesh rule, 1.0), DGR_CFG (c2 default; any synth config
name, e.g. c3 for the BL q=1 BBH).
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs, initial

t_end = float(sys.argv[1]) if len(sys.argv) > 1 else 100.0
samples = int(sys.argv[2]) if len(sys.argv) > 2 else 20
import dataclasses
from synth.configs import Puncture
lmax = int(os.environ.get("DGR_LMAX", "8"))
if os.environ.get("DGR_CFG", "c2") == "c2":
    cfg = configs.c2_schwarzschild(rho=float(os.environ.get("DGR_RHO", "1.0")), lmax=lmax)
else:
    cfg = configs.get(os.environ["DGR_CFG"])
if os.environ.get("DGR_PUNCT", "c2") == "cell":
    hh = cfg.width / (6.0 * (1 << lmax))
    cfg = dataclasses.replace(cfg, punctures=(Puncture(hh / 2, hh / 2, hh / 2, 1.0, lmax),))
m = dgr.Mesh(cfg)
xyz = m.dof_xyz_host()
n = xyz.shape[1]
u0 = initial.for_config(cfg, xyz, kind="bl")
sigma = float(os.environ.get("DGR_SIGMA", "0.4"))
eta = float(os.environ.get("DGR_ETA", "2.0"))
dt = float(os.environ.get("DGR_CFL", "0.25")) * m.info["h_min"]
bcs = {"both": (0, 1), "somm": (1,), "extrap": (0,)}[os.environ.get("DGR_BC", "both")]
steps = int(round(t_end / dt))
every = max(1, steps // samples)
r = np.sqrt((xyz ** 2).sum(axis=0))
far = torch.from_numpy(r > 0.75 * cfg.width / 2).cuda()   # outer region (near the boundary)
print(f"{cfg.name}: {m.info['n_oct_global']} octants, {n} DOFs, dt = {dt:.5f}, {steps} steps to t = {t_end}, "
      f"KO sigma {sigma}, eta {eta}")
for somm in bcs:
    prm = dgr.Params(sommerfeld=somm, ko_sigma=sigma, eta=eta,
                     upwind=int(os.environ.get("DGR_UPWIND", "0")))
    u = torch.zeros((24, m.dof_stride), dtype=torch.float64, device="cuda")
    u[:, :n] = torch.from_numpy(u0)
    print(f"--- outer boundary: {'Sommerfeld (R29)' if somm else 'extrapolation (R12)'}")
    print(f"{'t':>7s} {'H_L2':>10s} {'H_max':>10s} {'M_L2':>10s} {'G_L2':>10s} "
          f"{'H_max(outer)':>12s} {'alpha_min':>10s} {'finite':>6s}")
    t0 = time.time()
    for k in range(steps + 1):
        if k % every == 0 or k == steps:
            c, nm = m.constraints(u, prm=prm)
            fin = bool(torch.isfinite(u[:, :n]).all())
            hfar = float(c[0, :n][far].abs().max())
            mL2 = float(np.sqrt((nm[1:4, 0] ** 2).sum()))
            gL2 = float(np.sqrt((nm[4:7, 0] ** 2).sum()))
            print(f"{k * dt:7.2f} {nm[0, 0]:10.3e} {nm[0, 1]:10.3e} {mL2:10.3e} {gL2:10.3e} "
                  f"{hfar:12.3e} {float(u[0, :n].min()):10.5f} {str(fin):>6s}", flush=True)
            if not fin:
                break
        if k < steps:
            m.rk4_step(u, dt, prm=prm)
    torch.cuda.synchronize()
    print(f"    wall {time.time() - t0:.1f} s")
