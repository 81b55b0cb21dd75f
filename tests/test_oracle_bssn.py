"""Pins for oracle/bssn.py, oracle/constraints.py and oracle/rk4.py.

What the mathematics fixes (SURVEY.md §8c "What pins each part", Appendix A):
* Minkowski data -> RHS == 0 bitwise (through unzip, FD and zip).
* Ricci split (eqs 16-19, readings R1/R2/R3) == the Ricci tensor of
  gamma_ij = gt_ij / chi computed directly from its Christoffel symbols.
* Gauge wave (exact, time-dependent): with exact derivatives the algebra gives
  the exact d/dt of chi, K, Gt, beta, gt, At (1+log slicing is NOT the
  harmonic slicing of the gauge wave, so alpha and B are excluded — reading
  R27); with FD the error converges at O(h^6).
* Kerr-Schild (exact, stationary): d/dt of chi, K, Gt, gt, At vanishes with
  exact derivatives and converges to 0 at O(h^6) with FD; H, M^i, G^i vanish.
* Gauge-sector special cases that reduce to textbook ODEs, and invariance under
  a constant shift (Galilean advection) for every field.
* RK4: amplification 1 + z + z^2/2 + z^3/6 + z^4/24; temporal order 4.
"""
from types import SimpleNamespace

import numpy as np
import pytest
import sympy as sp

from oracle import bssn, constraints, fd, rk4
from oracle.maps import OracleMesh
from oracle.unzip import unzip
from synth import configs, initial
from synth.configs import MeshConfig, Puncture

from . import exact_solutions as ex
from .exact_solutions import X, Y, Z

PRM = bssn.Params()
GEOM = [1, 2, 3, 4, 5, 12, 13, 14, 15, 16, 17, 18, 19, 20, 21, 22, 23]   # chi K Gt gt At


def _pts(n, lo, hi, seed):
    return np.random.default_rng(seed).uniform(lo, hi, size=(3, n))


def test_minkowski_rhs_is_zero():
    m = OracleMesh(configs.small_adaptive(lmax=5, rho=0.5))
    u = initial.minkowski(m.dof_coords())
    r = rk4.rhs_dofs(m, u, PRM)
    assert np.all(r == 0.0)


# ------------------------------------------------------ exact-derivative pins

@pytest.fixture(scope="module")
def gw():
    return ex.gauge_wave()


@pytest.fixture(scope="module")
def ks():
    return ex.kerr_schild()


def test_gauge_wave_algebra_exact(gw):
    pts = _pts(7, 0.0, 1.0, 1)
    d = ex.pointdata(gw, pts)
    got = bssn.algebra(d, PRM)
    want = ex.time_derivative(gw, pts)
    idx = GEOM + [6, 7, 8]
    err = np.max(np.abs(got[idx] - want[idx]))
    assert err < 1e-12, err
    # the lapse really differs (1+log vs harmonic), so the check is not vacuous
    assert np.max(np.abs(got[0] - want[0])) > 1e-3


def test_kerr_schild_algebra_exact(ks):
    fields, _ = ks
    pts = _pts(6, 0.9, 1.8, 2) * np.array([[1], [-1], [1]])
    d = ex.pointdata(fields, pts)
    got = bssn.algebra(d, PRM)
    assert np.max(np.abs(got[GEOM])) < 1e-12
    c = constraints.constraints_point(d, PRM)
    assert np.max(np.abs(c)) < 1e-12
    # control: Lie weight 0 instead of -2/3 would leave an O(0.1) residual (Appendix A #7)
    assert np.max(np.abs(got[[0, 6, 7, 8]])) > 1e-3


def test_ricci_split_equals_direct_ricci():
    """R_ij = Rt_ij + Rchi_ij of eqs (16)-(19) vs the Ricci tensor of gt/chi."""
    a = [sp.Rational(k, 10) for k in (1, 2, -1, 3, 1, 2)]
    gt = sp.Matrix([[1 + a[0] * sp.sin(X + Y), a[1] * X * Z / 4, a[2] * sp.cos(Y)],
                    [a[1] * X * Z / 4, 1 + a[3] * sp.sin(Z) ** 2, a[4] * X * Y / 3],
                    [a[2] * sp.cos(Y), a[4] * X * Y / 3, 1 + a[5] * sp.cos(X - Z)]])
    chi = 1 / (1 + X ** 2 / 5 + Y * Z / 7)
    p = np.array([[0.31], [-0.42], [0.27]])
    ev = lambda e: float(e.subs({X: p[0, 0], Y: p[1, 0], Z: p[2, 0]}).evalf(30))
    # physical metric and its exact derivatives
    gam = gt / chi
    g0 = np.array([[ev(gam[i, j]) for j in range(3)] for i in range(3)])
    g1 = np.array([[[ev(sp.diff(gam[i, j], V)) for j in range(3)] for i in range(3)]
                   for V in ex.XYZ])                                     # [k, i, j]
    g2 = np.array([[[[ev(sp.diff(gam[i, j], A, B)) for j in range(3)] for i in range(3)]
                    for B in ex.XYZ] for A in ex.XYZ])                   # [k, l, i, j]
    gi = np.linalg.inv(g0)
    dgi = -np.einsum("ia,mab,bk->mik", gi, g1, gi)
    # Christoffel of the first kind [l, i, j] = 1/2(d_i g_lj + d_j g_li - d_l g_ij)
    Cl = 0.5 * (np.einsum("ilj->lij", g1) + np.einsum("jli->lij", g1) - g1)
    Gam = np.einsum("kl,lij->kij", gi, Cl)
    dCl = 0.5 * (np.einsum("milj->mlij", g2) + np.einsum("mjli->mlij", g2) - g2)  # [m, l, i, j]
    dGam = np.einsum("mkl,lij->mkij", dgi, Cl) + np.einsum("kl,mlij->mkij", gi, dCl)
    Ric = (np.einsum("kkij->ij", dGam) - np.einsum("jkik->ij", dGam)
           + np.einsum("kkl,lij->ij", Gam, Gam) - np.einsum("kjl,lik->ij", Gam, Gam))
    # BSSN inputs with Gt^i := CalGt^i = gt^ij gt^kl C_lij (exact values and
    # derivatives by the product rule from exact gt, d gt, dd gt)
    fields = [sp.Integer(1), chi, sp.Integer(0)] + [sp.Integer(0)] * 9 \
        + [gt[i, j] for (i, j) in ex.SYM] + [sp.Integer(0)] * 6
    d = ex.pointdata(fields, p)
    t0, t1, t2 = d.gt[..., 0], d.d_gt[..., 0], d.dd_gt[..., 0]
    ti = np.linalg.inv(t0)
    dti = -np.einsum("ia,mab,bk->mik", ti, t1, ti)
    C = 0.5 * (np.einsum("ilj->lij", t1) + np.einsum("jli->lij", t1) - t1)
    dC = 0.5 * (np.einsum("milj->mlij", t2) + np.einsum("mjli->mlij", t2) - t2)
    cal = np.einsum("ij,kl,lij->k", ti, ti, C)
    dcal = (np.einsum("mij,kl,lij->mk", dti, ti, C) + np.einsum("ij,mkl,lij->mk", ti, dti, C)
            + np.einsum("ij,kl,mlij->mk", ti, ti, dC))
    d.Gt = cal[:, None]
    d.d_Gt = dcal[..., None]
    G = bssn.geometry(d, PRM)
    err = np.max(np.abs(G["Ric"][..., 0] - Ric))
    assert err < 1e-11, err
    # the printed +1/2 sign (reading R1) would be off by O(0.1)
    alt = G["Ric"][..., 0] + np.einsum("lm,lmij->ij", G["ginv"][..., 0], d.dd_gt[..., 0])
    assert np.max(np.abs(alt - Ric)) > 1e-3


def _const_data(alpha=1.0, chi=1.0, K=0.0, beta=(0, 0, 0), B=(0, 0, 0)):
    z3, z33 = np.zeros((3, 1)), np.zeros((3, 3, 1))
    d = SimpleNamespace(alpha=np.array([alpha]), chi=np.array([chi]), K=np.array([K]),
                        Gt=z3.copy(), beta=np.array(beta, float)[:, None],
                        B=np.array(B, float)[:, None], gt=np.eye(3)[..., None].copy(),
                        At=z33.copy(), d_alpha=z3.copy(), d_chi=z3.copy(), d_K=z3.copy(),
                        d_Gt=z33.copy(), d_beta=z33.copy(), d_B=z33.copy(),
                        d_gt=np.zeros((3, 3, 3, 1)), d_At=np.zeros((3, 3, 3, 1)),
                        dd_alpha=z33.copy(), dd_chi=z33.copy(), dd_beta=np.zeros((3, 3, 3, 1)),
                        dd_gt=np.zeros((3, 3, 3, 3, 1)))
    return d


def test_gauge_sector_textbook_odes():
    a, k, c = 0.8, 0.3, 0.9
    prm = bssn.Params(eta=1.7, lambda_f0=0.6, lambda_f1=0.5)
    r = bssn.algebra(_const_data(alpha=a, chi=c, K=k, B=(0.2, -0.1, 0.4)), prm)[:, 0]
    assert r[0] == pytest.approx(-2 * a * k, rel=1e-14)              # 1+log: d_t a = -2 a K
    assert r[2] == pytest.approx(a * k * k / 3, rel=1e-14)           # d_t K = a K^2 / 3
    assert r[1] == pytest.approx(2 / 3 * c * a * k, rel=1e-14)        # d_t chi = 2/3 chi a K
    fa = 0.6 + 0.5 * a
    assert np.allclose(r[6:9], 0.75 * fa * np.array([0.2, -0.1, 0.4]), rtol=1e-14)  # Gamma-driver
    assert np.allclose(r[9:12], -1.7 * np.array([0.2, -0.1, 0.4]), rtol=1e-14)
    assert np.all(r[[3, 4, 5] + list(range(12, 24))] == 0)


def test_constant_shift_is_advection():
    """beta -> beta + b (constant b, Galilean boost of the coordinates' shift)
    adds exactly b.grad(f) to the RHS of EVERY field, beta's own included
    (eq 2: beta^j d_j beta^i; the transposed beta^j d_i beta^j would add
    b^j d_i beta^j instead) and B's (eq 3: the b.grad Gt that d_t Gt gains
    from eq 8 cancels against -beta^j d_j Gt^i, leaving b.grad B)."""
    cfg = MeshConfig(name="u2p", xmin=(0, 0, 0), width=1.0, periodic=True, level_min=2)
    m = OracleMesh(cfg)
    u = initial.random_smooth(m.dof_coords(), 1.0, seed=11)
    P0 = unzip(m, u)
    b = np.array([0.3, -0.2, 0.5])
    P1 = P0.copy()
    for i in range(3):
        P1[6 + i] = P0[6 + i] + b[i]
    h = rk4.octant_h(m)
    r0 = bssn.rhs_patches(P0, h, PRM)
    r1 = bssn.rhs_patches(P1, h, PRM)
    hh = h[:, None, None, None]
    assert np.max(np.abs(fd.grad(P0[6], hh))) > 1e-2          # beta really varies
    for f in range(24):
        g = fd.grad(P0[f], hh)
        want = b[0] * g[0] + b[1] * g[1] + b[2] * g[2]
        assert np.max(np.abs(r1[f] - r0[f] - want)) < 1e-11 * (1 + np.max(np.abs(want))), f


# ------------------------------------------------------------ FD convergence

def _uniform(width, xmin, level, periodic):
    return MeshConfig(name="u", xmin=xmin, width=width, periodic=periodic, level_min=level)


def test_gauge_wave_fd_convergence(gw):
    errs = []
    for level in (2, 3):
        m = OracleMesh(_uniform(1.0, (0.0, 0.0, 0.0), level, True))
        xyz = m.dof_coords()
        u = ex.values(gw, xyz)
        r = rk4.rhs_dofs(m, u, bssn.Params(ko_sigma=0.0))
        want = ex.time_derivative(gw, xyz)
        idx = GEOM + [6, 7, 8]
        errs.append(np.max(np.abs(r[idx] - want[idx])))
    order = np.log2(errs[0] / errs[1])
    assert order > 5.5, (errs, order)


def test_kerr_schild_fd_convergence(ks):
    fields, _ = ks
    errs, cerrs = [], []
    for level in (2, 3):
        m = OracleMesh(_uniform(2.0, (0.7, -2.4, 0.9), level, False))
        xyz = m.dof_coords()
        u = ex.values(fields, xyz)
        r = rk4.rhs_dofs(m, u, bssn.Params(ko_sigma=0.0))
        errs.append(np.max(np.abs(r[GEOM])))
        c = constraints.constraints_dofs(m, u, PRM)
        cerrs.append(np.max(np.abs(c)))
    # extrapolated outer boundary (reading R12): the padding is exact for degree
    # 6, so second derivatives next to the boundary are one-sided O(h^5)
    for e in (errs, cerrs):
        order = np.log2(e[0] / e[1])
        assert order > 4.5, (e, order)


def test_brill_lindquist_hamiltonian_converges():
    p = [Puncture(0.0, 0.0, 0.0, 1.0, 0)]
    errs = []
    for level in (2, 3):
        m = OracleMesh(_uniform(2.0, (0.8, 0.6, -1.0), level, False))
        u = initial.brill_lindquist(m.dof_coords(), p)
        c = constraints.constraints_dofs(m, u, PRM)
        assert np.all(c[1:4] == 0.0)        # K = At = 0 -> M^i = 0 exactly
        errs.append(np.max(np.abs(c[0])))
    order = np.log2(errs[0] / errs[1])
    assert order > 4.5, (errs, order)      # O(h^5) at the extrapolated boundary


# ---------------------------------------------------------------------- RK4

def test_rk4_amplification():
    for z in (-0.3, 0.2, -1.1 + 0.4j):
        lam = z
        out = rk4.rk4_step_generic(lambda v: lam * v, np.array([1.0 + 0j]), 1.0)[0]
        assert abs(out - (1 + z + z ** 2 / 2 + z ** 3 / 6 + z ** 4 / 24)) < 1e-15


def test_rk4_temporal_order():
    F = lambda v: -v * v + np.sin(v)
    def run(n):
        v = np.array([0.7])
        for _ in range(n):
            v = rk4.rk4_step_generic(F, v, 1.0 / n)
        return v[0]
    ref = run(4096)
    e1, e2 = abs(run(16) - ref), abs(run(32) - ref)
    assert 3.7 < np.log2(e1 / e2) < 4.3


# ------------------------------------------- shift-wave pins of eqs (2), (3), (8)

def _shift_wave(kvec, evec, eps):
    """Flat data (gt = delta, alpha = chi = 1, K = At = Gt = B = 0) with the
    shift plane wave beta^i = eps e^i sin(k.x): every term of eqs (1)-(8) is a
    closed form in e, k."""
    ph = sum(sp.Rational(kvec[a]) * V for a, V in enumerate(ex.XYZ))
    beta = [sp.Rational(eps) * sp.Rational(evec[i]) * sp.sin(ph) for i in range(3)]
    return ([sp.Integer(1), sp.Integer(1), sp.Integer(0)] + [sp.Integer(0)] * 3 + beta
            + [sp.Integer(0)] * 3
            + [sp.Integer(1 if i == j else 0) for (i, j) in ex.SYM] + [sp.Integer(0)] * 6), ph


def _closed_form_shift_wave(kvec, evec, eps, pts):
    k = np.array(kvec, float)
    e = np.array(evec, float)
    ph = np.einsum("a,an->n", k, pts)
    s, c = np.sin(ph), np.cos(ph)
    beta = eps * e[:, None] * s                       # [i, n]
    dbeta = eps * np.einsum("i,j->ji", e, k)[..., None] * c   # d_j beta^i -> [j, i, n]
    div = eps * (e @ k) * c
    return k, e, s, c, beta, dbeta, div


@pytest.mark.parametrize("kvec,evec", [((2, -1, 3), (1, 2, 0)),       # transverse: e.k = 0
                                       ((0, 3, -2), (5, 0, 0))])
def test_transverse_shift_wave(kvec, evec):
    """Transverse shift wave (e perpendicular to k): eq (2) gives
    d_t beta^i = beta^j d_j beta^i = eps^2 sin cos (e.k) e^i = 0 exactly (the
    transposed beta^j d_i beta^j would give eps^2 |e|^2 sin cos k^i); eq (8)
    gives d_t Gt^i = gt^jk d_j d_k beta^i = -|k|^2 beta^i (the divergence term
    vanishes, CalGt = 0); eq (3) then gives d_t B^i = d_t Gt^i = -|k|^2 beta^i
    (B = 0, Gt = 0).  P:L101 (eq 2), P:L103 (eq 3), P:L117-119 (eq 8)."""
    eps = sp.Rational(3, 10)
    fields, _ = _shift_wave(kvec, evec, eps)
    pts = _pts(5, -1.0, 1.0, 7)
    d = ex.pointdata(fields, pts)
    r = bssn.algebra(d, PRM)
    k, e, s, c, beta, dbeta, div = _closed_form_shift_wave(kvec, evec, float(eps), pts)
    assert e @ k == 0
    k2 = k @ k
    scale = 1 + k2
    assert np.max(np.abs(r[6:9])) < 1e-13 * scale                        # eq (2)
    assert np.max(np.abs(r[3:6] + k2 * beta)) < 1e-12 * scale            # eq (8)
    assert np.max(np.abs(r[9:12] + k2 * beta)) < 1e-12 * scale           # eq (3)
    # control: the transposed advection term is not small on these points
    transposed = np.einsum("jn,ijn->in", beta, dbeta)        # beta^j d_i beta^j
    assert np.max(np.abs(transposed)) > 1e-3
    # the rest of the system is closed form too: eq (4) Lie derivative of delta
    # (w = -2/3, div beta = 0): d_t gt_ij = d_i beta^j + d_j beta^i; eq (5) 0;
    # eqs (1), (6), (7): 0 (no curvature, alpha' = 0, K = At = 0)
    want_gt = np.stack([dbeta[j, i] + dbeta[i, j] for (i, j) in ex.SYM])
    assert np.max(np.abs(r[12:18] - want_gt)) < 1e-13 * scale
    assert np.max(np.abs(r[[0, 1, 2] + list(range(18, 24))])) < 1e-13 * scale


def test_longitudinal_shift_wave():
    """Longitudinal shift wave (e parallel to k): eq (8) gives
    d_t Gt^i = -|k|^2 beta^i - (1/3)|k|^2 beta^i = -(4/3)|k|^2 beta^i, eq (3)
    d_t B^i = the same, eq (2) d_t beta^i = eps^2 |k| sin cos khat^i, eq (5)
    d_t chi = -(2/3) div beta, eq (4) d_t gt_ij = 2 d_(i beta_j) - (2/3) delta_ij
    div beta.  P:L99-119."""
    kvec, evec = (1, 2, -2), (1, 2, -2)
    eps = sp.Rational(1, 5)
    fields, _ = _shift_wave(kvec, evec, eps)
    pts = _pts(5, -1.0, 1.0, 8)
    d = ex.pointdata(fields, pts)
    r = bssn.algebra(d, PRM)
    k, e, s, c, beta, dbeta, div = _closed_form_shift_wave(kvec, evec, float(eps), pts)
    k2 = k @ k
    scale = 1 + k2 * k2
    assert np.max(np.abs(r[3:6] + (4.0 / 3.0) * k2 * beta)) < 1e-12 * scale
    assert np.max(np.abs(r[9:12] + (4.0 / 3.0) * k2 * beta)) < 1e-12 * scale
    adv = np.einsum("jn,jin->in", beta, dbeta)                # beta^j d_j beta^i
    assert np.max(np.abs(r[6:9] - adv)) < 1e-13 * scale
    assert np.max(np.abs(adv)) > 1e-3
    assert np.max(np.abs(r[1] + (2.0 / 3.0) * div)) < 1e-13 * scale
    want_gt = np.stack([dbeta[j, i] + dbeta[i, j] - (2.0 / 3.0) * (i == j) * div
                        for (i, j) in ex.SYM])
    assert np.max(np.abs(r[12:18] - want_gt)) < 1e-13 * scale


def test_b_equation_couples_to_gt_evolution():
    """Eq (3) with a nonzero, varying Gt^i and shift: d_t B^i - d_t Gt^i =
    -eta B^i + beta^j d_j B^i - beta^j d_j Gt^i exactly, whatever the rest of
    eq (8) is.  Deleting the d_t Gt - beta.grad Gt coupling, or the
    beta.grad B term, fails."""
    rng = np.random.default_rng(5)
    c = [sp.Rational(int(v), 10) for v in rng.integers(-9, 10, size=12)]
    Gt = [c[0] * sp.sin(X + 2 * Y), c[1] * sp.cos(Z - X), c[2] * X * Y]
    beta = [c[3] + c[4] * sp.sin(Y), c[5] + c[6] * Z * X, c[7] + c[8] * sp.cos(X + Z)]
    B = [c[9] * sp.cos(Y + Z), c[10] * X * X, c[11] * sp.sin(Z)]
    gt = [1 + X * Y / 10, Z / 20, 0, 1 + sp.sin(X) / 10, Y / 30, 1]
    fields = [1 + X / 10, 1 + Y * Z / 10, X * Z / 5] + Gt + beta + B + gt \
        + [X / 10, 0, Y / 10, Z / 10, 0, X * Y / 10]
    fields = [sp.sympify(f) for f in fields]
    pts = _pts(6, -0.5, 0.5, 9)
    d = ex.pointdata(fields, pts)
    prm = bssn.Params(eta=1.3)
    r = bssn.algebra(d, prm)
    adv = lambda g: np.einsum("jn,jin->in", d.beta, g)
    want = -1.3 * d.B + adv(d.d_B) - adv(d.d_Gt)
    assert np.max(np.abs((r[9:12] - r[3:6]) - want)) < 1e-13
    assert np.max(np.abs(r[3:6])) > 1e-2          # d_t Gt is not trivially zero here
    assert np.max(np.abs(adv(d.d_Gt))) > 1e-3
