"""Quick timing of one RK4 step (device-resident) on a config; not the bench."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs, initial
name = sys.argv[1] if len(sys.argv) > 1 else "c3"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
cfg = configs.get(name)
fused = os.environ.get("DGR_FUSED", "1") != "0"
t = time.time(); m = dgr.Mesh(cfg); m.set_fused(fused); print("fused", fused)
print("mesh", m.info, "%.1fs" % (time.time() - t), flush=True)
xyz = m.dof_xyz_host()
u = torch.zeros((24, m.dof_stride), dtype=torch.float64, device="cuda")
u[:, :xyz.shape[1]] = torch.from_numpy(initial.for_config(cfg, xyz))
dt = 0.25 * m.info["h_min"]
for _ in range(2): m.rk4_step(u, dt)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(steps): m.rk4_step(u, dt)
e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / steps
n = m.info["n_dof_owned"]; no = m.info["n_oct_local"]
print(f"{name}: {ms:.3f} ms/step, {n/ms*1e3:.3e} DOF-steps/s, {no*343/ms*1e3:.3e} oct-pts/s, launches/step {m.last_launch_count()}")
r = m.rhs(u); torch.cuda.synchronize()
e0.record()
for _ in range(steps): m.rhs(u, out=r)
e1.record(); torch.cuda.synchronize()
print(f"{name}: rhs (unzip+rhs+zip) {e0.elapsed_time(e1)/steps:.3f} ms")
m.profile_read(reset=True); m.profile_enable(True)
for _ in range(2): m.rk4_step(u, dt)
torch.cuda.synchronize(); m.profile_enable(False)
for k, (t, n) in m.profile_read(reset=True).items():
    print(f"  {k:12s} {t/n:8.3f} ms/launch  {n:4d} launches  {t/2:8.3f} ms/step")
print("finite:", bool(torch.isfinite(u[:, :n]).all()))
