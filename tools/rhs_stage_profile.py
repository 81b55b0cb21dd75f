"""Per-stage cycle profile of k_rhs (experiment build: DGR_LIB=.../libdgr_timing.so)."""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs, initial
cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "c3")
m = dgr.Mesh(cfg)
m.set_fused(os.environ.get("DGR_FUSED", "1") != "0")
xyz = m.dof_xyz_host()
u = torch.zeros((24, m.dof_stride), dtype=torch.float64, device="cuda")
u[:, :xyz.shape[1]] = torch.from_numpy(initial.for_config(cfg, xyz))
m.rhs(u); torch.cuda.synchronize()
buf = (C.c_longlong * 25)()
dgr.lib().dgr_debug_rhs_stage_cycles(buf)
m.rhs(u); torch.cuda.synchronize()
dgr.lib().dgr_debug_rhs_stage_cycles(buf)
order = [12, 13, 14, 15, 16, 17, 1, 0, 3, 4, 5, 6, 7, 8, 2, 18, 19, 20, 21, 22, 23, 9, 10, 11]
names = ["alpha", "chi", "K", "Gt0", "Gt1", "Gt2", "b0", "b1", "b2", "B0", "B1", "B2",
         "gxx", "gxy", "gxz", "gyy", "gyz", "gzz", "Axx", "Axy", "Axz", "Ayy", "Ayz", "Azz"]
v = np.array(buf[:], dtype=np.float64)
tot = v.sum()
print("slot 0 = epilogue-to-prologue gap; slot k = stage k-1; slot 24 = stage 23")
lab = ["(prologue)"] + [names[order[k]] + (" +CH" if k == 5 else "") for k in range(24)]
for k in range(25):
    print(f"{k:3d} {lab[k]:12s} {100 * v[k] / tot:6.2f}%")
