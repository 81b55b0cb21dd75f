"""Sensitivity of 100 RK4 steps to a 1e-13 relative perturbation (GPU, libdgr).
Tells whether 1e-8 parity after 100 steps is attainable for a setup."""
import sys, os, dataclasses
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs, initial
from synth.configs import MeshConfig, Puncture
cases = {
  "tiny_bl": (MeshConfig(name="tiny", xmin=(-4.,-4.,-4.), width=8.0, periodic=False, level_min=1, punctures=(Puncture(0.1,-0.2,0.05,1.0,4),), rho=0.4), "bl"),
  "small_bl": (configs.small_adaptive(lmax=5, rho=0.5), "bl"),
  "c2_bl": (configs.c2_schwarzschild(), "bl"),
  "u2_gw": (MeshConfig(name="u2", xmin=(-.5,-.5,-.5), width=1.0, periodic=True, level_min=2), "gauge_wave"),
  "c1_gw": (configs.c1_uniform(), "gauge_wave"),
  "c1_rand": (configs.c1_uniform(), "random"),
  "bbh_small": (configs.small_bbh(lmax=6, rho=0.5), "bl"),
  "bbh_small_rand": (configs.small_bbh(lmax=6, rho=0.5), "random"),
  "bbh5_bl": (configs.small_bbh(lmax=5, rho=0.4), "bl"),
  "bbh5_rand": (configs.small_bbh(lmax=5, rho=0.4), "random"),
  "small_rand": (configs.small_adaptive(lmax=5, rho=0.5), "random"),
  # smooth constraint-satisfying data (gauge wave, A = 0.1, one wavelength
  # across the domain) on the adaptive puncture meshes (mesh from the
  # punctures, data independent of them)
  "bbh_small_gw": (configs.small_bbh(lmax=6, rho=0.5), "gauge_wave"),
  "bbh5_gw": (configs.small_bbh(lmax=5, rho=0.4), "gauge_wave"),
  "small_gw": (configs.small_adaptive(lmax=5, rho=0.5), "gauge_wave"),
  "bbh_small_gw_per": (dataclasses.replace(configs.small_bbh(lmax=6, rho=0.5), periodic=True), "gauge_wave"),
}
only = sys.argv[1:]
if only:
    cases = {k: v for k, v in cases.items() if k in only}
for name, (cfg, kind) in cases.items():
    m = dgr.Mesh(cfg)
    xyz = m.dof_xyz_host(); n = xyz.shape[1]
    u0 = initial.for_config(cfg, xyz, kind=kind, seed=3)
    rng = np.random.default_rng(0)
    ua = torch.zeros((24, m.dof_stride), dtype=torch.float64, device="cuda"); ua[:, :n] = torch.from_numpy(u0)
    ub = ua.clone(); ub[:, :n] *= torch.from_numpy(1 + 1e-13 * rng.standard_normal(u0.shape)).cuda()
    dt = 0.25 * m.info["h_min"]
    out = []
    for k in range(100):
        m.rk4_step(ua, dt); m.rk4_step(ub, dt)
        if (k + 1) in (1, 10, 25, 50, 100):
            a, b = ua[:, :n], ub[:, :n]
            rel = ((a - b).abs().amax(1) / a.abs().amax(1).clamp_min(1e-300)).max().item()
            out.append(f"{k+1}:{rel:.1e}")
    finite = bool(torch.isfinite(ua).all())
    print(f"{name:10s} oct={m.info['n_oct_global']:6d} maxabs={ua[:, :n].abs().max().item():.3e} finite={finite} rel-diff " + " ".join(out), flush=True)
