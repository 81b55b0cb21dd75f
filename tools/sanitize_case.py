"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck):
every libdgr kernel of the hot path on small_bbh (hanging chains, extrapolated
boundary) — fused stage (k_interp, k_gt_pre, k_rhs, k_rk4), two-pass path
(k_unzip, k_rhs on patches, k_zip_rk4), radiative boundary, constraints, and
the group exchange (k_pack, k_unpack) with 2 rank-meshes on one device."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_fernandonhzsgb22_b200 as dgr  # noqa: E402
from synth import configs, initial  # noqa: E402

lmax = int(sys.argv[1]) if len(sys.argv) > 1 else 5
cfg = configs.small_bbh(lmax=lmax, rho=0.4)
m = dgr.Mesh(cfg)
xyz = m.dof_xyz_host()
u = initial.for_config(cfg, xyz)
ud = m.new_state()
ud[:, :xyz.shape[1]] = torch.from_numpy(u).cuda()
dt = 0.25 * m.info["h_min"]
m.rk4_step(ud, dt)
m.rhs(ud, prm=dgr.Params(sommerfeld=1))
m.set_fused(False)
m.rk4_step(ud, dt)
m.set_fused(True)
m.constraints(ud)
meshes = [dgr.Mesh(cfg, rank=r, nranks=2) for r in range(2)]
sts = []
for mm in meshes:
    gid = mm.export(dgr.MAP_DOF_GID, np.int64)
    st = mm.new_state()
    st[:, :mm.info["n_dof_owned"]] = torch.from_numpy(u[:, gid[:mm.info["n_dof_owned"]]]).cuda()
    sts.append(st)
g = dgr.Group(meshes)
g.rk4_step(sts, dt)
torch.cuda.synchronize()
g.close()
# regrid (k_wavelet, k_transfer) and Psi_4 extraction (k_rhs_inputs, k_psi4,
# k_sphere_interp), lopsided advection, generated algebra kernels
w = m.regrid_indicator(ud).cpu().numpy()
octs = m.regrid_octree(w, float(np.quantile(w, 0.8)), float(np.quantile(w, 0.3)), 1, lmax + 1)
m2 = dgr.Mesh(cfg, octs)
m.regrid_transfer(ud, m2)
m.psi4_modes(ud, (0.013, -0.021, 0.007), 5.0, 6, 12, l_max=3)
m.rk4_step(ud, dt, prm=dgr.Params(upwind=1))
inp = m.rhs_inputs(ud)
for v in dgr.ALG_VARIANTS:
    dgr.rhs_algebra(v, inp)
torch.cuda.synchronize()
print("sanitize case done", flush=True)
