"""Pins for oracle/fd.py and the interpolation tables of oracle/unzip.py.

What the mathematics fixes (SURVEY.md §8c "What pins each part"):
* D1 is exact for polynomials of degree <= 6 and D2 for degree <= 7; the first
  non-exact monomials give D1(x^7)(0) = 36 h^6 and D2(x^8)(0) = 72 h^6.
* D_xy = D1_x D1_y is exact on x^a y^b for a, b <= 6.
* Observed convergence order 6 on smooth functions under h-halving.
* KO annihilates polynomials of degree <= 5; on the Nyquist mode it gives
  -sigma/h * u (dissipative); PAPER.md L95 only says "KO dissipation".
* Lagrange rows are dyadic (golden values, tests/golden/stencils.txt).
"""
import os
from fractions import Fraction

import numpy as np
import pytest

from oracle import fd, unzip

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "stencils.txt")


def _grid(h):
    t = (np.arange(13) - 6) * h        # patch centre at 0, interior index 3..9
    z, y, x = np.meshgrid(t, t, t, indexing="ij")
    return x, y, z


def _patch(fun, h):
    x, y, z = _grid(h)
    return fun(x, y, z)[None]          # [1, 13, 13, 13]


def _interior_xyz(h):
    x, y, z = _grid(h)
    s = slice(3, 10)
    return x[s, s, s], y[s, s, s], z[s, s, s]


@pytest.mark.parametrize("a", [0, 1, 2])
@pytest.mark.parametrize("deg", range(0, 7))
def test_d1_exact_to_degree6(a, deg):
    h = 0.37
    P = _patch(lambda x, y, z: [x, y, z][a] ** deg + 0.3 * [y, z, x][a], h)
    xi = _interior_xyz(h)
    exact = deg * xi[a] ** (deg - 1) if deg else 0.0 * xi[a]
    got = fd.d1(P, a, np.array(h).reshape(1, 1, 1, 1))[0]
    assert np.max(np.abs(got - exact)) < 1e-9 * max(1.0, np.max(np.abs(exact)))


@pytest.mark.parametrize("a", [0, 1, 2])
@pytest.mark.parametrize("deg", range(0, 8))
def test_d2_exact_to_degree7(a, deg):
    h = 0.41
    P = _patch(lambda x, y, z: [x, y, z][a] ** deg, h)
    xi = _interior_xyz(h)
    exact = deg * (deg - 1) * xi[a] ** (deg - 2) if deg >= 2 else 0.0 * xi[a]
    got = fd.d2(P, a, np.array(h).reshape(1, 1, 1, 1))[0]
    assert np.max(np.abs(got - exact)) < 1e-8 * max(1.0, np.max(np.abs(exact)))


def test_first_nonexact_monomials():
    h = 0.5
    hh = np.array(h).reshape(1, 1, 1, 1)
    P7 = _patch(lambda x, y, z: x ** 7, h)
    P8 = _patch(lambda x, y, z: x ** 8, h)
    # the centre of the patch (index 6) is interior point (3,3,3)
    assert fd.d1(P7, 0, hh)[0, 3, 3, 3] == pytest.approx(36 * h ** 6, rel=1e-12)
    assert fd.d2(P8, 0, hh)[0, 3, 3, 3] == pytest.approx(72 * h ** 6, rel=1e-12)


@pytest.mark.parametrize("a,b", [(0, 1), (0, 2), (1, 2), (1, 0)])
def test_mixed_exact(a, b):
    h = 0.29
    rng = np.random.default_rng(1)
    pa, pb = rng.integers(0, 7, size=2)
    f = lambda x, y, z: [x, y, z][a] ** pa * [x, y, z][b] ** pb
    P = _patch(f, h)
    xi = _interior_xyz(h)
    va, vb = xi[a], xi[b]
    exact = (pa * va ** (pa - 1) if pa else 0 * va) * (pb * vb ** (pb - 1) if pb else 0 * vb)
    got = fd.dmixed(P, a, b, np.array(h).reshape(1, 1, 1, 1))[0]
    assert np.max(np.abs(got - exact)) < 1e-8 * max(1.0, np.max(np.abs(exact)))


def test_hess_symmetric_and_matches_mixed():
    h = 0.1
    P = _patch(lambda x, y, z: np.sin(x + 2 * y) * np.cos(z - x), h)
    H = fd.hess(P, np.array(h).reshape(1, 1, 1, 1))
    assert np.array_equal(H[0, 1], H[1, 0])
    assert np.allclose(fd.dmixed(P, 1, 0, np.array(h).reshape(1, 1, 1, 1)), H[0, 1], rtol=1e-12, atol=1e-12)


def test_sixth_order_convergence():
    f = lambda x, y, z: np.sin(1.3 * x + 0.7) * np.exp(0.4 * y) * np.cos(0.9 * z)
    fx = lambda x, y, z: 1.3 * np.cos(1.3 * x + 0.7) * np.exp(0.4 * y) * np.cos(0.9 * z)
    fxx = lambda x, y, z: -1.69 * f(x, y, z)
    fxz = lambda x, y, z: -0.9 * 1.3 * np.cos(1.3 * x + 0.7) * np.exp(0.4 * y) * np.sin(0.9 * z)
    errs = {"d1": [], "d2": [], "dxz": []}
    for h in (0.08, 0.04):
        P = _patch(f, h)
        hh = np.array(h).reshape(1, 1, 1, 1)
        xi = _interior_xyz(h)
        errs["d1"].append(np.max(np.abs(fd.d1(P, 0, hh)[0] - fx(*xi))))
        errs["d2"].append(np.max(np.abs(fd.d2(P, 0, hh)[0] - fxx(*xi))))
        errs["dxz"].append(np.max(np.abs(fd.dmixed(P, 0, 2, hh)[0] - fxz(*xi))))
    for k, (e0, e1) in errs.items():
        order = np.log2(e0 / e1)
        # pure stencils converge at exactly 6; the product D1 D1 of a separable
        # function has its h^6 terms partly cancel at the max-error point here
        assert 5.6 < order < (6.6 if k != "dxz" else 7.5), (k, order)


@pytest.mark.parametrize("deg", range(0, 6))
def test_ko_annihilates_degree5(deg):
    h = 0.3
    P = _patch(lambda x, y, z: x ** deg + y ** deg - 2 * z ** deg, h)
    got = fd.ko_sum(P, np.array(h).reshape(1, 1, 1, 1), 0.4)
    assert np.max(np.abs(got)) < 1e-10


def test_ko_nyquist_is_dissipative():
    h, sigma = 0.25, 0.4
    i = np.arange(13)
    v = (-1.0) ** i
    P = np.broadcast_to(v[None, None, :], (13, 13, 13))[None].copy()
    got = fd.ko(P, 0, np.array(h).reshape(1, 1, 1, 1), sigma)[0]
    expect = -(sigma / h) * v[3:10][None, None, :]
    assert np.allclose(got, np.broadcast_to(expect, got.shape), rtol=1e-14)


def _golden():
    out = {}
    with open(GOLDEN) as fh:
        for line in fh:
            line = line.split("#")[0].strip()
            if not line:
                continue
            key, vals = line.split(":")
            out[key.strip()] = [Fraction(v) for v in vals.split()]
    return out


def test_lagrange_rows_golden():
    g = _golden()
    W = unzip.W13
    # unit rows at integer t
    for t in range(7):
        e = np.zeros(7)
        e[t] = 1.0
        assert np.array_equal(W[2 * t], e)
    for t2, key in ((1, "interp_t_1/2"), (3, "interp_t_3/2"), (5, "interp_t_5/2")):
        assert [Fraction(x) for x in W[t2]] == g[key]
    for t, key in enumerate(("extrap_t_-1", "extrap_t_-2", "extrap_t_-3")):
        assert [Fraction(x) for x in unzip.WEXT[t]] == g[key]
    # mirror symmetry l_m(t) = l_{6-m}(6-t)
    for t2 in range(13):
        assert np.array_equal(W[t2], W[12 - t2][::-1])
    assert np.allclose(W.sum(axis=1), 1.0, rtol=0, atol=1e-15)


def test_fd_weights_golden():
    """The stencils applied to unit impulses reproduce the golden weights."""
    g = _golden()
    h = 1.0
    hh = np.array(h).reshape(1, 1, 1, 1)
    w1, w2, wk = [], [], []
    for s in range(-3, 4):
        P = np.zeros((1, 13, 13, 13))
        P[0, 6, 6, 6 + s] = 1.0
        w1.append(Fraction(fd.d1(P, 0, hh)[0, 3, 3, 3] * 60).limit_denominator(1))
        w2.append(Fraction(fd.d2(P, 0, hh)[0, 3, 3, 3] * 180).limit_denominator(1))
        wk.append(Fraction(fd.ko(P, 0, hh, 64.0)[0, 3, 3, 3]).limit_denominator(1))
    assert w1 == g["d1_times_60"]
    assert w2 == g["d2_times_180"]
    assert wk == g["ko_times_64h_over_sigma"]


# ------------------------------------------------ lopsided advection (R9u)

def test_lopsided_stencils_exact_to_degree4_and_upwind_side():
    """oracle.fd.lop_plus / lop_minus (reading R9u): exact first derivative of
    polynomials of degree <= 4 (4th order), first error at x^5 with the
    closed-form coefficient; the plus stencil reads offsets -1..3 only (a
    perturbation at -2 or -3 leaves it unchanged), the minus one -3..1; and
    fd.advect picks the side by the sign of beta^a."""
    from oracle import fd as _fd
    h = 0.125
    z = np.arange(13) - 6.0                         # patch index -> x / h, interior centre at 0
    X = np.broadcast_to((z * h)[None, None, :], (13, 13, 13)).copy()
    for deg in range(5):
        P = X ** deg
        want = deg * X[3:10, 3:10, 3:10] ** max(deg - 1, 0) if deg else 0 * X[3:10, 3:10, 3:10]
        assert np.abs(_fd.lop_plus(P, 0, h) - want).max() < 1e-12
        assert np.abs(_fd.lop_minus(P, 0, h) - want).max() < 1e-12
    # x^5 at x = 0: plus (-3(-1) - 0 + 18 - 6*32 + 243)/12 h^4 = 6 h^4; minus
    # (3 + 0 + 18 - 6*32 + 243)/12 h^4 = 6 h^4 (odd function, mirrored stencil)
    P = X ** 5
    c = (6, 6)
    assert abs(_fd.lop_plus(P, 0, h)[c + (3,)] - 6.0 * h ** 4) < 1e-12
    assert abs(_fd.lop_minus(P, 0, h)[c + (3,)] - 6.0 * h ** 4) < 1e-12
    Q = np.zeros((13, 13, 13))
    Q[:, :, 6 - 2] = 1.0                            # offset -2 of interior point x = 3 (index 6)
    assert _fd.lop_plus(Q, 0, h)[:, :, 3].max() == 0.0
    assert _fd.lop_minus(Q, 0, h)[:, :, 3].max() != 0.0
    rng = np.random.default_rng(0)
    U = rng.standard_normal((13, 13, 13))
    beta = np.stack([np.where(rng.uniform(size=(7, 7, 7)) > 0.5, 1.0, -1.0) * 0.3,
                     np.zeros((7, 7, 7)), np.zeros((7, 7, 7))])
    got = _fd.advect(U, beta, h, True)
    want = beta[0] * np.where(beta[0] >= 0, _fd.lop_plus(U, 0, h), _fd.lop_minus(U, 0, h))
    assert np.array_equal(got, want)
    assert np.array_equal(_fd.advect(U, beta, h, False), beta[0] * _fd.d1(U, 0, h))


def test_upwind_rhs_reduces_to_centred_where_fields_are_linear():
    """With every field linear in x (lopsided and centred stencils are both exact
    on degree <= 1, up to rounding), the upwind RHS equals the centred one; on
    generic data they differ."""
    from oracle import bssn as _b, rk4 as _rk4
    from oracle.maps import OracleMesh
    from oracle.unzip import unzip
    from synth.configs import MeshConfig
    cfg = MeshConfig(name="lin", xmin=(-1, -1, -1), width=2.0, periodic=False, level_min=1)
    m = OracleMesh(cfg)
    m.build_dofs()
    x = m.dof_coords()
    rng = np.random.default_rng(3)
    a, b = rng.uniform(-0.1, 0.1, 24), rng.uniform(-0.05, 0.05, (24, 3))
    base = np.zeros(24)
    base[[0, 1, 12, 15, 17]] = 1.0
    u = base[:, None] + a[:, None] + b @ x
    P = unzip(m, u)
    h = _rk4.octant_h(m)
    r0 = _b.rhs_patches(P, h, _b.Params(ko_sigma=0.0))
    r1 = _b.rhs_patches(P, h, _b.Params(ko_sigma=0.0, upwind=1))
    assert np.abs(r1 - r0).max() < 1e-12 * (1 + np.abs(r0).max())
    u2 = u + 0.05 * np.sin(3.0 * x[0])[None, :]
    P2 = unzip(m, u2)
    d = np.abs(_b.rhs_patches(P2, h, _b.Params(upwind=1)) - _b.rhs_patches(P2, h, _b.Params()))
    assert d.max() > 1e-6
