"""Where does the C2 instability start?  Position (radius) and value of
max |H| and of max |rhs| per field group along the run (diagnostic)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs, initial
cfg = configs.c2_schwarzschild(rho=float(os.environ.get("DGR_RHO", "1.0")))
prm = dgr.Params(upwind=int(os.environ.get("DGR_UPWIND", "0")),
                 ko_sigma=float(os.environ.get("DGR_SIGMA", "0.4")))
m = dgr.Mesh(cfg)
xyz = m.dof_xyz_host(); n = xyz.shape[1]
r = np.sqrt((xyz ** 2).sum(axis=0))
u = torch.zeros((24, m.dof_stride), dtype=torch.float64, device="cuda")
u[:, :n] = torch.from_numpy(initial.for_config(cfg, xyz, kind="bl"))
dt = 0.25 * m.info["h_min"]
names = ["alpha", "chi", "K", "Gt", "beta", "B", "gt", "At"]
groups = [[0], [1], [2], [3, 4, 5], [6, 7, 8], [9, 10, 11], list(range(12, 18)), list(range(18, 24))]
for k in range(0, 1200):
    if k % 96 == 0:
        c, nm = m.constraints(u, prm=prm)
        H = c[0, :n].abs().cpu().numpy()
        i = int(np.argmax(H))
        rh = m.rhs(u, prm=prm)[:, :n].abs().cpu().numpy()
        chi = u[1, :n].cpu().numpy()
        al = u[0, :n].cpu().numpy()
        print(f"      chi_min={chi.min():.3e}@r={r[np.argmin(chi)]:.3f}  alpha_min={al.min():.3e}@r={r[np.argmin(al)]:.3f}"
              f"  alpha(r<0.1)max={al[r < 0.1].max():.3e}", flush=True)
        s = " ".join(f"{nm_}:{rh[g].max():.1e}@r={r[np.unravel_index(np.argmax(rh[g]), rh[g].shape)[1]]:.2f}"
                     for nm_, g in zip(names, groups))
        print(f"t={k*dt:6.2f} |H|max={H[i]:.2e} at r={r[i]:.3f}  {s}", flush=True)
        if not np.isfinite(H).all():
            break
    m.rk4_step(u, dt, prm=prm)
