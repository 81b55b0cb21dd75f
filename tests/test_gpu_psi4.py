"""GPU parity of gravitational-wave extraction (readings R33-R36, SURVEY
§8(f) row 4) against oracle/psi4.py through the C ABI: Psi_4 at every octant
node (generated k_psi4 over the 234 derivative inputs), its interpolation to
extraction-sphere points and the (l, m) modes, within 1e-10."""
import numpy as np
import pytest

import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from oracle import psi4 as op4
from oracle.maps import OracleMesh
from synth import configs, initial

from .gpu_util import need_gpu, to_dev, torch

pytestmark = pytest.mark.gpu
CENTER = (0.013, -0.021, 0.007)        # off the node lattice: no node on the tetrad's axis


@pytest.fixture(scope="module")
def setup():
    need_gpu()
    cfg = configs.small_bbh(lmax=4, rho=0.4)
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords(), kind="random", seed=9)
    m = dgr.Mesh(cfg)
    return cfg, om, u, m, to_dev(u, m.dof_stride)


def test_psi4_octant_nodes(setup):
    cfg, om, u, m, ud = setup
    got = m.psi4(ud, CENTER).cpu().numpy()
    want = op4.psi4_octants(om, u, CENTER).reshape(-1)
    scale = np.abs(want).max()
    assert np.isfinite(got).all() and scale > 1e-3
    assert np.abs(got[0] - want.real).max() <= 1e-10 * scale
    assert np.abs(got[1] - want.imag).max() <= 1e-10 * scale


def test_psi4_sphere_and_modes(setup):
    cfg, om, u, m, ud = setup
    radius, nt, npf = 9.0, 10, 20
    modes, sph = m.psi4_modes(ud, CENTER, radius, nt, npf, l_max=4)
    xyz, T, P, W = op4.sphere_points(radius, nt, npf, CENTER)
    vals = op4.psi4_octants(om, u, CENTER)
    want_s, _ = op4.interpolate(om, vals, xyz)
    scale = np.abs(want_s).max()
    assert np.abs(sph[0] + 1j * sph[1] - want_s).max() <= 1e-10 * scale
    want = op4.modes(want_s, T, P, W, l_max=4)
    mscale = max(abs(v) for v in want.values())
    for k, v in want.items():
        assert abs(modes[k] - v) <= 1e-10 * mscale, (k, modes[k], v)
