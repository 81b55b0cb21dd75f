"""Table II / Fig. 11 of the paper redone on one B200.

For a mesh config: the derivatives-through-HBM path — dgr_rhs_inputs (unzip +
one derivative kernel writing the 234 inputs of A per point) followed by each
generated A kernel (SymPyGR CSE, binary reduce, staged CSE; natural and
occupancy-constrained builds) — against the fused hand-staged kernels
(k_gt_pre + k_rhs) on the same state.  CUDA events; prints one JSON line.

    python tools/codegen_bench.py [config] [reps]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_fernandonhzsgb22_b200 as dgr  # noqa: E402
from synth import configs, initial  # noqa: E402


def timed(fn, reps):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "c3"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    cfg = configs.get(name)
    m = dgr.Mesh(cfg)
    xyz = m.dof_xyz_host()
    u = m.new_state()
    u[:, :xyz.shape[1]] = torch.from_numpy(initial.for_config(cfg, xyz)).cuda()
    npts = m.info["n_oct_local"] * 343
    res = {"config": name, "octants": m.info["n_oct_local"], "points": npts}
    inp = m.rhs_inputs(u)
    m.profile_enable(True)
    m.profile_read(reset=True)
    res["inputs_total_ms"] = timed(lambda: m.rhs_inputs(u, out=inp), reps)
    prof = m.profile_read(reset=True)
    res["inputs_kernels_ms"] = {k: v[0] / v[1] for k, v in prof.items()}
    out = torch.empty((24, npts), dtype=torch.float64, device="cuda")
    for v in dgr.ALG_VARIANTS:
        for occ in (False, True):
            ms = timed(lambda: dgr.rhs_algebra(v, inp, occ=occ, out=out), reps)
            res[f"{v}{'_occ4' if occ else ''}_ms"] = ms
            res[f"{v}{'_occ4' if occ else ''}_ns_per_point"] = ms * 1e6 / npts
    # the fused hand-staged path on the same state: derivatives never stored
    r = m.new_state()
    m.profile_read(reset=True)
    res["fused_rhs_total_ms"] = timed(lambda: m.rhs(u, out=r), reps)
    prof = m.profile_read(reset=True)
    res["fused_kernels_ms"] = {k: v[0] / v[1] for k, v in prof.items()}
    m.profile_enable(False)
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
