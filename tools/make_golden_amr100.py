"""Expected state for the AMR 100-step parity test (tests/test_gpu_parity.py::
test_100_steps_amr_golden), written by the ORACLE ONLY (oracle/ + synth/).

north_star: RK4 state within 1e-8 of the oracle after 100 steps; BASELINE
configs[1] asks for it on an adaptive mesh.  The oracle needs ~400 RHS
evaluations on this mesh (tens of minutes), too slow for the GPU test suite,
so the state is computed once here and committed: a seeded sample of the DOFs
(all 24 fields) plus per-field max-abs and RMS over ALL DOFs.

    python tools/make_golden_amr100.py [name]      (DGR_ORACLE_WORKERS = cores)
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

from oracle import bssn, rk4  # noqa: E402
from oracle.maps import OracleMesh  # noqa: E402
from synth import configs, initial  # noqa: E402

CASES = {
    # small_bbh: q = 2 BBH, levels 2..6 on [-16,16]^3, 428 octants, hanging
    # chains, extrapolated outer boundary, Brill-Lindquist data
    "small_bbh_bl": (lambda: configs.small_bbh(lmax=6, rho=0.5), "bl"),
}
STEPS = 100
NSAMPLE = 6000


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "small_bbh_bl"
    cfgf, kind = CASES[name]
    cfg = cfgf()
    om = OracleMesh(cfg)
    om.build_dofs()
    u0 = initial.for_config(cfg, om.dof_coords(), kind=kind, seed=5)
    dt = rk4.dt_courant(om)
    prm = bssn.Params()
    v = u0.copy()
    t0 = time.time()
    for k in range(STEPS):
        v = rk4.rk4_step(om, v, dt, prm)
        if (k + 1) % 10 == 0:
            print(f"step {k + 1}: {time.time() - t0:.0f} s, max|u| {np.abs(v).max():.6e}", flush=True)
    idx = np.sort(np.random.default_rng(2024).choice(om.n_dof, size=min(NSAMPLE, om.n_dof),
                                                     replace=False))
    out = os.path.join(ROOT, "tests", "golden", f"amr100_{name}.npz")
    np.savez_compressed(out, idx=idx, u=v[:, idx], fmax=np.abs(v).max(axis=1),
                        frms=np.sqrt((v * v).mean(axis=1)), dt=dt, steps=STEPS,
                        n_oct=om.n_oct, n_dof=om.n_dof, kind=kind, seed=5,
                        moved=np.abs(v - u0).max())
    print("wrote", out, "max|u100 - u0|", np.abs(v - u0).max())


if __name__ == "__main__":
    main()
