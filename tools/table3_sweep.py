"""Table III of the paper on one B200: octant-to-patch (unzip)
and patch-to-octant (zip) on five puncture meshes of decreasing adaptivity
m1..m5 (BL q=1, finest level 12, 10, 8, 6, 4; synth.configs.table3_mesh).
Per mesh: octants, the interpolation-slot kernel, the two-pass k_unzip (13^3
patches of 24 fields written to HBM), the zip gather k_zip (RHS per octant
point -> DOFs), each with its algorithmic bytes and the fraction of the
measured HBM bandwidth.  One JSON line per mesh.

    python tools/table3_sweep.py [reps]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_fernandonhzsgb22_b200 as dgr  # noqa: E402
from synth import configs, initial  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6650.0}
HBM = peaks["hbm_gbs"]
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 5
for k in range(1, 6):
    cfg = configs.table3_mesh(k)
    m = dgr.Mesh(cfg)
    xyz = m.dof_xyz_host()
    u = m.new_state()
    u[:, :xyz.shape[1]] = torch.from_numpy(initial.for_config(cfg, xyz)).cuda()
    no, nd = m.info["n_oct_local"], m.info["n_dof_owned"]
    P = m.unzip(u)
    m.set_zip_store(False)
    r = m.rhs(u)
    torch.cuda.synchronize()
    m.profile_enable(True)
    m.profile_read(reset=True)
    for _ in range(reps):
        m.unzip(u, patches=P)
    pu = m.profile_read(reset=True)
    for _ in range(reps):
        m.rhs(u, out=r)
    pz = m.profile_read(reset=True)
    m.profile_enable(False)
    ms = lambda d, c: d[c][0] / d[c][1] if c in d else None
    t_unzip, t_interp, t_zip = ms(pu, "unzip"), ms(pu, "interp"), ms(pz, "zip_rk4")
    b_unzip = 24 * (2197 + 216) * 8 * no              # write every patch point, read every DOF once
    b_interp = 24 * 8 * m.info["n_interp_slots"] + (24 * 343 * 8 + 343 * 4) * m.info["n_interp_elems"]
    b_zip = 24 * nd * (8 + 8) + nd * 4                 # read the owner's value, write the DOF, zip map
    res = {"mesh": cfg.name, "levels": [m.info["level_min"], m.info["level_max"]], "octants": no,
           "dofs": nd, "interp_slots": m.info["n_interp_slots"],
           "unzip_ms": t_unzip, "unzip_GBps": b_unzip / t_unzip / 1e6, "unzip_frac": b_unzip / t_unzip / 1e6 / HBM,
           "interp_ms": t_interp,
           "interp_GBps": b_interp / t_interp / 1e6 if t_interp else None,
           "zip_ms": t_zip, "zip_GBps": b_zip / t_zip / 1e6, "zip_frac": b_zip / t_zip / 1e6 / HBM,
           "hbm_peak_GBps": HBM}
    print(json.dumps(res), flush=True)
