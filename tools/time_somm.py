"""C3 RK4 step time with the radiative outer boundary (dgr_params.sommerfeld) and
the lopsided advection (dgr_params.upwind) vs the default (CUDA events, graph replay)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs, initial
cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "c3")
m = dgr.Mesh(cfg)
xyz = m.dof_xyz_host()
u = m.new_state()
u[:, :xyz.shape[1]] = torch.from_numpy(initial.for_config(cfg, xyz)).cuda()
dt = 0.25 * m.info["h_min"]
for name, prm in (("extrapolated (R12)", None), ("sommerfeld (R29)", dgr.Params(sommerfeld=1)),
                  ("extrapolated + lopsided advection (R9u)", dgr.Params(upwind=1)),
                  ("sommerfeld + lopsided advection", dgr.Params(sommerfeld=1, upwind=1))):
    for _ in range(3):
        m.rk4_step(u, dt, prm=prm)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        m.rk4_step(u, dt, prm=prm)
    e1.record(); torch.cuda.synchronize()
    print(f"{name}: {e0.elapsed_time(e1) / 10:.3f} ms/step")
