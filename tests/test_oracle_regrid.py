"""Pins for oracle/regrid.py (readings R30-R32; Alg. 1 line 3,
P:L198-215) and the C++ regrid octree against it.

What the mathematics fixes:
* the wavelet indicator vanishes (to rounding) on data that are polynomials of
  degree <= 6 per axis (the degree-6 prediction reproduces them), is of the
  size of the degree-7 term otherwise, and equals a brute-force evaluation of
  its definition on one octant;
* the transfer reproduces polynomials of degree <= 6 per axis on any pair of
  meshes, is the identity (bitwise) from a mesh to itself, and refine-then-
  coarsen returns the original DOF values bitwise (coarsening only copies);
* the regridded octree is complete, 2:1 balanced, Morton sorted, refines every
  leaf above the tolerance and changes every leaf by at most one level.
The C++ builder (dgr_regrid_octree) gives the oracle's octree bit-for-bit.
"""
from fractions import Fraction

import numpy as np
import pytest

from oracle import octree, regrid
from oracle.maps import OracleMesh
from oracle.unzip import lagrange_weights, unzip
from synth import configs, initial

CFG = configs.small_bbh(lmax=4, rho=0.4)


@pytest.fixture(scope="module")
def mesh():
    m = OracleMesh(CFG)
    m.build_dofs()
    return m


def _poly(xyz, deg):
    x, y, z = (xyz[a] / 16.0 for a in range(3))
    base = 1.0 + x ** deg - 0.5 * y ** (deg - 1) * z + 0.25 * x * y * z ** (deg - 2)
    return np.stack([base * (1 + 0.1 * f) for f in range(24)])


def test_indicator_zero_on_degree6(mesh):
    u = _poly(mesh.dof_coords(), 6)
    w = regrid.wavelet_indicator(mesh, u)
    assert w.max() < 1e-12 * np.abs(u).max(), w.max()
    u7 = _poly(mesh.dof_coords(), 7)
    assert regrid.wavelet_indicator(mesh, u7).max() > 1e-6


def test_indicator_bruteforce_one_octant(mesh):
    u = initial.for_config(CFG, mesh.dof_coords(), kind="random", seed=2)
    w = regrid.wavelet_indicator(mesh, u)
    e = int(np.argmax(w))
    P = unzip(mesh, u, np.array([e]))[:, 0]                  # [f, z, y, x]
    best = 0.0
    for iz in range(3, 10):
        for iy in range(3, 10):
            for ix in range(3, 10):
                def row(i):
                    if i % 2 == 0:
                        r = [0.0] * 7
                        r[i // 2] = 1.0
                        return r
                    return [float(v) for v in lagrange_weights(Fraction(i, 2))]
                rx, ry, rz = row(ix), row(iy), row(iz)
                for f in range(24):
                    pred = sum(rz[c] * ry[b] * rx[a] * P[f, 2 * c, 2 * b, 2 * a]
                               for c in range(7) for b in range(7) for a in range(7))
                    best = max(best, abs(P[f, iz, iy, ix] - pred))
    assert abs(best - w[e]) <= 1e-12 * max(best, 1e-300), (best, w[e])


def _regridded(mesh, u):
    w = regrid.wavelet_indicator(mesh, u)
    er, ec = np.quantile(w, 0.8), np.quantile(w, 0.3)
    a, l = regrid.new_octree(mesh, w, er, ec, 1, 6)
    return w, er, ec, a, l


def test_new_octree_properties(mesh):
    u = initial.for_config(CFG, mesh.dof_coords(), kind="random", seed=1)
    w, er, ec, a, l = _regridded(mesh, u)
    D = mesh.D
    assert octree.is_complete(a, l, D)
    keys = octree.morton_key(a[:, 0], a[:, 1], a[:, 2], D)
    assert np.all(np.diff(keys) > 0)
    nm = OracleMesh(CFG, a, l)
    # every old leaf is covered by new leaves at most one level apart
    for e in range(mesh.n_oct):
        X = 6 * mesh.anchors[e] + 3 * mesh.side[e]          # old leaf centre
        c = nm.loc.leaf_of_cell(*(X // 6))
        assert abs(int(nm.levels[c]) - int(mesh.levels[e])) <= 1
        if w[e] > er and mesh.levels[e] < 6:
            assert nm.levels[c] == mesh.levels[e] + 1
    assert len(l) != mesh.n_oct                              # it did change


def test_balance_bruteforce_tiny():
    from synth.configs import MeshConfig, Puncture
    cfg = MeshConfig(name="t", xmin=(-1, -1, -1), width=2.0, periodic=False, level_min=1,
                     punctures=(Puncture(0.3, -0.2, 0.1, 1.0, 3),), rho=0.3)
    m = OracleMesh(cfg)
    m.build_dofs()
    rng = np.random.default_rng(0)
    w = rng.uniform(0, 1, m.n_oct)
    a, l = regrid.new_octree(m, w, 0.7, 0.4, 1, 4)
    assert octree.is_balanced_bruteforce(a, l, m.D, False)


def test_transfer_polynomial_identity_roundtrip(mesh):
    u = initial.for_config(CFG, mesh.dof_coords(), kind="random", seed=1)
    _, _, _, a, l = _regridded(mesh, u)
    nm = OracleMesh(CFG, a, l)
    nm.build_dofs()
    p6 = _poly(mesh.dof_coords(), 6)
    got = regrid.transfer(mesh, p6, nm)
    want = _poly(nm.dof_coords(), 6)
    assert np.abs(got - want).max() < 1e-12 * np.abs(want).max()
    assert np.array_equal(regrid.transfer(mesh, u, mesh), u)
    # refine every leaf once, then merge every family back: bitwise roundtrip
    fine_a, fine_l = octree.children(mesh.anchors, mesh.levels, mesh.D)
    fine_a, fine_l = octree.sort_morton(fine_a, fine_l, mesh.D)
    fm = OracleMesh(CFG, fine_a, fine_l)
    fm.build_dofs()
    uf = regrid.transfer(mesh, u, fm)
    back_a, back_l = regrid.new_octree(fm, np.zeros(fm.n_oct), 1.0, 0.5, 0, 20)
    assert np.array_equal(back_a, mesh.anchors) and np.array_equal(back_l, mesh.levels)
    assert np.array_equal(regrid.transfer(fm, uf, mesh), u)


@pytest.mark.parametrize("cfgf", [lambda: configs.small_bbh(lmax=4, rho=0.4),
                                  lambda: configs.small_adaptive(lmax=5, rho=0.5)])
def test_cpp_regrid_octree_matches_oracle(cfgf):
    import paper_conf_sc_fernandonhzsgb22_b200 as dgr
    cfg = cfgf()
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords(), kind="random", seed=4)
    w = regrid.wavelet_indicator(om, u)
    for q in ((0.8, 0.3), (0.5, 0.5), (0.95, 0.05)):
        er, ec = np.quantile(w, q[0]), np.quantile(w, q[1])
        a, l = regrid.new_octree(om, w, er, ec, 2, 7)
        m = dgr.Mesh(cfg, device=False)
        got = m.regrid_octree(w, er, ec, 2, 7)
        assert np.array_equal(got[:, :3].astype(np.int64), a), q
        assert np.array_equal(got[:, 3].astype(np.int64), l), q
