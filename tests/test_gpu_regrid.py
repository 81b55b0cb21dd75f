"""GPU parity of the regrid kernels (readings R30-R32)
against oracle/regrid.py, through the C ABI: the wavelet indicator (1e-10 of
its largest value on periodic data; on a non-periodic mesh the boundary
octants' predictions use extrapolated padding, whose rounding is amplified by
the extrapolation rows — same conditioning bound as the unzip parity test),
the intergrid transfer (1e-10 per field; bitwise identity to the same mesh and
bitwise refine-then-coarsen roundtrip)."""
import dataclasses

import numpy as np
import pytest

import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from oracle import octree, regrid
from oracle.maps import OracleMesh
from synth import configs, initial

from .gpu_util import assert_parity, need_gpu, to_dev, torch

pytestmark = pytest.mark.gpu


def _setup(cfg, seed=1):
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords(), kind="random", seed=seed)
    m = dgr.Mesh(cfg)
    return om, u, m, to_dev(u, m.dof_stride)


def test_indicator_parity_periodic():
    need_gpu()
    cfg = dataclasses.replace(configs.small_bbh(lmax=5, rho=0.4), periodic=True)
    om, u, m, ud = _setup(cfg)
    w = m.regrid_indicator(ud).cpu().numpy()
    wo = regrid.wavelet_indicator(om, u)
    assert np.abs(w - wo).max() <= 1e-10 * wo.max(), np.abs(w - wo).max() / wo.max()


def test_indicator_parity_extrapolated_boundary():
    need_gpu()
    cfg = configs.small_bbh(lmax=5, rho=0.4)
    om, u, m, ud = _setup(cfg)
    w = m.regrid_indicator(ud).cpu().numpy()
    wo = regrid.wavelet_indicator(om, u)
    n = 1 << om.D
    bnd = np.any((om.anchors == 0) | (om.anchors + om.side[:, None] == n), axis=1)
    err = np.abs(w - wo)
    assert err[~bnd].max() <= 1e-10 * wo.max()
    # boundary octants: the prediction reads extrapolated padding points; each
    # extrapolation pass amplifies rounding by sum|w_t| <= 2815 (t = 3), so two
    # implementations agree to 8 eps * 2815^3 * max|u| at worst
    assert err[bnd].max() <= 8 * 2.2e-16 * 2815.0 ** 3 * np.abs(u).max()


def test_transfer_parity_and_identities():
    need_gpu()
    cfg = configs.small_bbh(lmax=5, rho=0.4)
    om, u, m, ud = _setup(cfg, seed=3)
    wo = regrid.wavelet_indicator(om, u)
    er, ec = np.quantile(wo, 0.8), np.quantile(wo, 0.3)
    octs = m.regrid_octree(wo, er, ec, 2, 7)
    a, l = regrid.new_octree(om, wo, er, ec, 2, 7)
    assert np.array_equal(octs[:, :3].astype(np.int64), a)
    nm_o = OracleMesh(cfg, a, l)
    nm_o.build_dofs()
    nm = dgr.Mesh(cfg, octs)
    assert nm.info["n_dof_owned"] == nm_o.n_dof
    un = m.regrid_transfer(ud, nm)[:, :nm_o.n_dof].cpu().numpy()
    assert_parity(un, regrid.transfer(om, u, nm_o), 1e-10, "regrid transfer")
    # identity to the same mesh, bitwise
    same = m.regrid_transfer(ud, dgr.Mesh(cfg))
    assert torch.equal(same[:, :om.n_dof], ud[:, :om.n_dof])
    # refine every leaf, transfer, merge back, transfer: bitwise roundtrip
    fa, fl = octree.children(om.anchors, om.levels, om.D)
    fa, fl = octree.sort_morton(fa, fl, om.D)
    fine = dgr.Mesh(cfg, np.concatenate([fa, fl[:, None]], axis=1).astype(np.uint32))
    uf = m.regrid_transfer(ud, fine)
    back = fine.regrid_octree(np.zeros(fine.info["n_oct_global"]), 1.0, 0.5, 0, 18)
    assert np.array_equal(back, m.octants)
    ub = fine.regrid_transfer(uf, dgr.Mesh(cfg, back))
    assert torch.equal(ub[:, :om.n_dof], ud[:, :om.n_dof])
