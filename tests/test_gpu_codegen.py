"""GPU parity of the generated RHS-algebra kernels (the
paper's Table II variants) against the oracle, through the C ABI:
every variant (SymPyGR CSE, binary reduce, staged CSE), natural and
occupancy-constrained builds, within 1e-10 per field; and the whole
derivatives-through-HBM path (dgr_rhs_inputs + dgr_rhs_algebra) on an
adaptive mesh against the oracle's RHS and against the fused k_rhs."""
import numpy as np
import pytest

import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from oracle import bssn as obssn
from oracle import rk4 as ork4
from oracle import unzip as ouz
from oracle.maps import OracleMesh
from synth import configs, initial

from .codegen_util import oracle_rhs, random_inputs, relerr
from .gpu_util import need_gpu, to_dev, torch

pytestmark = pytest.mark.gpu
TOL = 1e-10


@pytest.mark.parametrize("variant", dgr.ALG_VARIANTS)
@pytest.mark.parametrize("occ", [False, True])
def test_generated_algebra_random(variant, occ):
    need_gpu()
    x = random_inputs(5000, seed=11)
    prm = dgr.Params(eta=1.7, lambda_f0=0.8, lambda_f1=0.3, chi_floor=0.6)
    out = dgr.rhs_algebra(variant, torch.from_numpy(x).cuda(), prm, occ=occ).cpu().numpy()
    want = oracle_rhs(x, obssn.Params(eta=1.7, lambda_f0=0.8, lambda_f1=0.3, chi_floor=0.6))
    err = relerr(out, want)
    assert err.max() < TOL, (variant, occ, err)


def test_inputs_plus_generated_algebra_on_mesh():
    need_gpu()
    cfg = configs.small_bbh(lmax=5, rho=0.4)
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords(), kind="random", seed=3)
    m = dgr.Mesh(cfg)
    ud = to_dev(u, m.dof_stride)
    inp = m.rhs_inputs(ud)
    want = obssn.rhs_patches(ouz.unzip(om, u), ork4.octant_h(om), obssn.Params()).reshape(24, -1)
    fused = m.rhs_patches(m.unzip(ud)).reshape(24, -1).cpu().numpy()
    assert relerr(fused, want).max() < TOL
    for v in dgr.ALG_VARIANTS:
        got = dgr.rhs_algebra(v, inp).cpu().numpy()
        assert relerr(got, want).max() < TOL, v
