"""Pins for oracle/unzip.py (octant-to-patch, Alg. 2).

* Polynomial reproduction: any p(x) q(y) r(z) with per-axis degree <= 6 sampled
  at the DOFs unzips to its exact values at all 2197 points of every patch on
  balanced adaptive trees (copy, injection, interpolation, hanging chains and
  outer-boundary extrapolation are all exact for such data).  A degree-7 factor
  is not reproduced (the check can fail).
* Uniform periodic tree: every patch point is a bitwise copy of the DOF at the
  wrapped position.
* zip(unzip(u)) = u bitwise on the DOFs (patch-to-octant).
"""
import numpy as np
import pytest

from oracle import unzip as ouz
from oracle.maps import K, KIND_INTERP, OracleMesh, _patch_ijk
from synth import configs
from synth.configs import MeshConfig, Puncture


def _poly(coef, t):
    return sum(c * t ** k for k, c in enumerate(coef))


def _patch_coords(m):
    pijk = _patch_ijk()
    X = 6 * m.anchors[:, None, :] + (pijk[None] - K) * m.side[:, None, None]
    unit = m.cfg.width / m.L
    return [m.cfg.xmin[a] + X[..., a] * unit for a in range(3)]          # [n, 2197]


def _chain_mesh():
    return configs.small_bbh(lmax=6, rho=0.5)


@pytest.mark.parametrize("cfgf", [lambda: configs.small_adaptive(lmax=5, rho=0.5),
                                  _chain_mesh])
def test_polynomial_reproduction(cfgf):
    cfg = cfgf()
    m = OracleMesh(cfg)
    m.build_dofs()
    rng = np.random.default_rng(7)
    xyz = m.dof_coords()
    s = cfg.width / 2
    c = rng.uniform(-1, 1, size=(3, 7))
    f = lambda x, y, z: _poly(c[0], x / s) * _poly(c[1], y / s) * _poly(c[2], z / s)
    u = np.stack([f(*xyz), 2.0 + f(*xyz) * 0.5])
    P = ouz.unzip(m, u).reshape(2, m.n_oct, -1)
    px = _patch_coords(m)
    exact = f(*px)
    src, kind = m.padding_sources()
    ext = (kind & 7) == 4
    scale = np.max(np.abs(exact))
    err_in = np.max(np.abs(P[0] - exact)[~ext]) / scale
    assert err_in < 1e-13, err_in
    # extrapolation rows at t=-3 have sum|w| = 2815 and corner points are
    # extrapolated three times in sequence, so rounding grows up to
    # eps * 2815^3 ~ 2e-6 of the stencil values; a wrong weight/index is O(1)
    err_ext = np.max(np.abs(P[0] - exact)[ext]) / scale
    assert err_ext < 1e-7, err_ext
    # the mesh really exercised interpolation and extrapolation
    assert np.any((kind & 7) == KIND_INTERP) and np.any((kind & 7) == 4)


def test_degree7_not_reproduced():
    m = OracleMesh(configs.small_adaptive(lmax=5, rho=0.5))
    m.build_dofs()
    xyz = m.dof_coords()
    f = lambda x, y, z: (x / 8.0) ** 7 + 0 * y
    P = ouz.unzip(m, f(*xyz)[None]).reshape(m.n_oct, -1)
    px = _patch_coords(m)
    assert np.max(np.abs(P - f(*px))) > 1e-8


def test_hanging_chains_present():
    """Coarser sources whose own interpolation stencil holds hanging points."""
    m = OracleMesh(_chain_mesh())
    m.build_dofs()
    ht = m.hanging_table()
    srcs = np.unique(ht[:, 2])
    has_hanging = (~m.is_dof[srcs]).any(axis=1)
    assert has_hanging.any()


def test_uniform_periodic_copies():
    cfg = configs.c1_uniform()
    m = OracleMesh(cfg)
    m.build_dofs()
    xyz = m.dof_coords()
    rng = np.random.default_rng(3)
    u = rng.standard_normal((2, m.n_dof))
    P = ouz.unzip(m, u).reshape(2, m.n_oct, -1)
    # lattice position of every patch point, wrapped, -> DOF id via a dictionary
    unit = cfg.width / m.L
    lut = {tuple(np.rint((xyz[:, d] - np.array(cfg.xmin)) / unit).astype(np.int64) % m.L): d
           for d in range(m.n_dof)}
    pijk = _patch_ijk()
    for b in range(0, m.n_oct, 37):
        X = (6 * m.anchors[b] + (pijk - K) * m.side[b]) % m.L
        ids = np.array([lut[tuple(x)] for x in X])
        assert np.array_equal(P[:, b, :], u[:, ids])


@pytest.mark.parametrize("name", ["small", "c1"])
def test_zip_unzip_identity(name):
    cfg = configs.small_adaptive(lmax=5, rho=0.5) if name == "small" else configs.c1_uniform()
    m = OracleMesh(cfg)
    m.build_dofs()
    rng = np.random.default_rng(5)
    u = rng.standard_normal((3, m.n_dof))
    P = ouz.unzip(m, u)
    inner = P[:, :, K:K + 7, K:K + 7, K:K + 7].reshape(3, m.n_oct, 343)
    assert np.array_equal(ouz.zip_rhs(m, inner), u)
