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
v = np.array(buf[:], dtype=np.float64)
tot = v.sum()
# default path (fused, metric pre-pass, light-field pairs; rhs_kernel.cu c_stg_pre):
# slot 0 = epilogue of the previous octant + prologue (values, pre-pass rows,
# Christoffel block); slot k = stage k-1; slot 24 = the last stage
stages = ["chi", "alpha", "b0", "b1", "b2", "Gt0", "Gt1+Gt2", "K+Axx", "Axy+Axz", "Ayy+Ayz",
          "Azz+B0", "B1+B2"]
print("slot 0 = epilogue-to-prologue (incl. Christoffel block); slot k = stage k-1")
for k in range(len(stages) + 1):
    lab = "(prologue)" if k == 0 else stages[k - 1]
    val = v[k] if k < len(stages) else v[k] + v[24]
    print(f"{k:3d} {lab:12s} {100 * val / tot:6.2f}%")
print(f"cycles total {tot:.3e} (CTA thread 0, summed over octants)")
