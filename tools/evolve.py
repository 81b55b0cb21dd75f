"""Alg. 1 of the paper end to end on one GPU: evolve a
puncture data set with RK4 steps on the device, re-grid every f_r steps
(wavelet indicator -> new octree on the host -> intergrid transfer, readings
R30-R32), extract Psi_4 modes on a sphere every `extract_every` steps
(R33-R36: "e.g. every 16 timesteps") and monitor the
constraints.  Prints one line per extraction: t, the (2,2) and (2,0) modes,
H_L2, octants.

    python tools/evolve.py [config=c3] [t_end=60] [radius=40]
Environment: DGR_FR (re-grid frequency in steps, 400), DGR_EPS_R / DGR_EPS_C
(wavelet tolerances, 1e-2 / 1e-6), DGR_EXTRACT (16).
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_fernandonhzsgb22_b200 as dgr  # noqa: E402
from synth import configs, initial  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c3"
t_end = float(sys.argv[2]) if len(sys.argv) > 2 else 60.0
radius = float(sys.argv[3]) if len(sys.argv) > 3 else 40.0
fr = int(os.environ.get("DGR_FR", "400"))
eps_r = float(os.environ.get("DGR_EPS_R", "1e-2"))
eps_c = float(os.environ.get("DGR_EPS_C", "1e-6"))
every = int(os.environ.get("DGR_EXTRACT", "16"))
cfg = configs.get(name)
prm = dgr.Params(sommerfeld=1)
m = dgr.Mesh(cfg)
xyz = m.dof_xyz_host()
u = m.new_state()
u[:, :xyz.shape[1]] = torch.from_numpy(initial.for_config(cfg, xyz)).cuda()
dt = 0.25 * m.info["h_min"]
lmin, lmax = m.info["level_min"], m.info["level_max"]
steps = int(round(t_end / dt))
print(f"{name}: {m.info['n_oct_global']} octants, dt {dt:.5f}, {steps} steps, regrid every {fr}, "
      f"extract every {every} at r = {radius}", flush=True)
print(f"{'t':>7s} {'Re C22':>11s} {'Im C22':>11s} {'|C20|':>10s} {'H_L2':>10s} {'octants':>8s} "
      f"{'Re C20':>11s}")
t0 = time.time()
t_regrid = 0.0
for k in range(steps + 1):
    if k % every == 0 or k == steps:
        modes, _ = m.psi4_modes(u, (0.0, 0.0, 0.0), radius, 16, 32, l_max=3, prm=prm)
        _, nm = m.constraints(u, prm=prm)
        c22, c20 = modes[(2, 2)], modes[(2, 0)]
        print(f"{k * dt:7.2f} {c22.real: .4e} {c22.imag: .4e} {abs(c20):.4e} {nm[0, 0]:.4e} "
              f"{m.info['n_oct_global']:8d} {c20.real: .4e}", flush=True)
        if not np.isfinite(nm[0, 0]):
            break
    if k > 0 and k % fr == 0 and k < steps:
        # Alg. 1 line 3: construct_grid(u) — the only host round trip
        tr = time.time()
        w = m.regrid_indicator(u).cpu().numpy()
        octs = m.regrid_octree(w, eps_r, eps_c, lmin, lmax)
        if len(octs) != m.info["n_oct_global"] or not np.array_equal(octs, m.octants):
            m2 = dgr.Mesh(cfg, octs)
            u2 = m.regrid_transfer(u, m2)
            m, u = m2, u2
            print(f"# regrid at t = {k * dt:.2f}: {len(octs)} octants "
                  f"(w max {w.max():.2e}, {time.time() - tr:.1f} s)", flush=True)
        t_regrid += time.time() - tr
    if k < steps:
        m.rk4_step(u, dt, prm)
torch.cuda.synchronize()
print(f"# wall {time.time() - t0:.1f} s (regrid {t_regrid:.1f} s)")
