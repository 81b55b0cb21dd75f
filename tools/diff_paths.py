"""Per-field differences between the fused and two-pass RHS (debug helper)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs, initial
cfg = configs.small_bbh(lmax=5, rho=0.4)
m = dgr.Mesh(cfg)
xyz = m.dof_xyz_host()
for kind in ("bl", "random"):
    u = initial.for_config(cfg, xyz, kind=kind, seed=6)
    if kind == "bl":
        u[6:9] = 0.2 * np.sin((xyz[0] + 2.0 * xyz[1] - xyz[2]) / 3.0 + np.arange(3)[:, None])
    ud = torch.zeros((24, m.dof_stride), dtype=torch.float64, device="cuda")
    ud[:, :xyz.shape[1]] = torch.from_numpy(u)
    for up in (0, 1):
        for pre in (True, False):
            m.set_prepass(pre)
            m.set_fused(True)
            r = m.rhs(ud, prm=dgr.Params(upwind=up))
            m.set_fused(False)
            r2 = m.rhs(ud, prm=dgr.Params(upwind=up))
            m.set_fused(True)
            d = (r - r2).abs().amax(dim=1).cpu().numpy()
            print(kind, "upwind", up, "prepass", pre, "fields differing:", [(f, float(d[f])) for f in range(24) if d[f] > 0])
        m.set_prepass(True)
