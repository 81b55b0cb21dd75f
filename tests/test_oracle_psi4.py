"""Pins for oracle/psi4.py (readings R33-R36).

What the mathematics fixes:
* Schwarzschild (Kerr-Schild slice, exact derivatives): the radial tetrad's
  null directions are the principal ones, so Psi_4 = 0 although E_ij and B_ij
  are not;
* a linearised TT plane wave along z: Psi_4 = (E - iB)(mbar, mbar) with
  E_ij = -h''_ij / 2 and B_ij = eps_izl h''_lj / 2 (closed forms from h), on
  the z axis -h''_+ + i h''_x — to O(eps^2);
* spin-weighted harmonics: Goldberg's closed forms for l = 2 and
  orthonormality under the product quadrature;
* the sphere interpolation reproduces degree-6 data; a synthetic Psi_4 built
  from known modes gives them back.
"""
import numpy as np
import pytest
import sympy as sp

from oracle import psi4
from oracle.maps import OracleMesh
from synth import configs

from . import exact_solutions as ex
from .exact_solutions import X, Y, Z


def _offaxis_points(n, rmin, rmax, seed):
    rng = np.random.default_rng(seed)
    r = rng.uniform(rmin, rmax, n)
    th = rng.uniform(0.3, np.pi - 0.3, n)
    ph = rng.uniform(0, 2 * np.pi, n)
    return np.stack([r * np.sin(th) * np.cos(ph), r * np.sin(th) * np.sin(ph), r * np.cos(th)])


def test_schwarzschild_psi4_vanishes():
    fields, _ = ex.kerr_schild()
    pts = _offaxis_points(6, 2.0, 5.0, 1)
    d = ex.pointdata(fields, pts)
    p4 = psi4.psi4_point(d, pts)
    assert np.max(np.abs(p4)) < 1e-12
    # not vacuous: the electric part is the tidal field ~ M / r^3
    from oracle import bssn
    G = bssn.geometry(d, bssn.Params())
    assert np.max(np.abs(G["Ric"])) > 1e-3


def _plane_wave(eps, w):
    u = -Z                                                     # t - z at t = 0
    hp, hx = sp.sin(w * u), sp.Rational(1, 2) * sp.cos(w * u)
    h = sp.Matrix([[hp, hx, 0], [hx, -hp, 0], [0, 0, 0]])
    gamma = sp.eye(3) + eps * h
    T = sp.Symbol("t")
    ht = h.subs(Z, Z - T)                                     # h(t - z)
    Kij = -sp.Rational(1, 2) * eps * sp.diff(ht, T).subs(T, 0)
    return ex.bssn_from_adm(gamma, sp.Integer(1), [0, 0, 0], Kij), (hp, hx)


def test_linearised_plane_wave_psi4():
    eps, w = sp.Rational(1, 10 ** 6), sp.Rational(3, 2)
    fields, (hp, hx) = _plane_wave(eps, w)
    pts = _offaxis_points(5, 1.0, 3.0, 2)
    d = ex.pointdata(fields, pts)
    got = psi4.psi4_point(d, pts)
    # closed forms: h'' (second derivative in u = t - z), E = -h''/2, B_ij = eps_izl h''_lj / 2
    ev = lambda e: np.array([float(e.subs(Z, z)) for z in pts[2]])
    hpp = [ev(sp.diff(hp, Z, 2)), ev(sp.diff(hx, Z, 2))]     # d^2/du^2 = d^2/dz^2
    H = np.zeros((3, 3, pts.shape[1]))
    H[0, 0], H[1, 1], H[0, 1], H[1, 0] = hpp[0], -hpp[0], hpp[1], hpp[1]
    H *= float(eps)
    E = -0.5 * H
    Bh = 0.5 * np.einsum("il,ljn->ijn", psi4.PERM[:, 2, :], H)
    B = 0.5 * (Bh + np.einsum("ijn->jin", Bh))
    _, et, ep = psi4.tetrad(pts, np.broadcast_to(np.eye(3)[..., None], (3, 3, pts.shape[1])))
    mb = (et - 1j * ep) / np.sqrt(2.0)
    want = np.einsum("in,ijn,jn->n", mb, E - 1j * B, mb)
    scale = float(eps) * float(w) ** 2
    assert np.max(np.abs(got - want)) < 1e-4 * scale        # O(eps^2) / O(eps)
    assert np.max(np.abs(want)) > 0.1 * scale
    # on (near) the +z axis: Psi_4 = -h''_+ + i h''_x
    pz = np.array([[1e-7], [0.0], [1.7]])
    dz = ex.pointdata(fields, pz)
    onaxis = psi4.psi4_point(dz, pz)[0]
    hpz = float(eps) * np.array([float(sp.diff(hp, Z, 2).subs(Z, 1.7)),
                                 float(sp.diff(hx, Z, 2).subs(Z, 1.7))])
    assert abs(onaxis - (-hpz[0] + 1j * hpz[1])) < 1e-4 * scale


def test_swsh_closed_forms_and_orthonormality():
    rng = np.random.default_rng(0)
    th, ph = rng.uniform(0, np.pi, 9), rng.uniform(0, 2 * np.pi, 9)
    c = np.cos(th)
    assert np.allclose(psi4.swsh(-2, 2, 2, th, ph), np.sqrt(5 / (64 * np.pi)) * (1 + c) ** 2 * np.exp(2j * ph), atol=1e-14)
    assert np.allclose(psi4.swsh(-2, 2, -2, th, ph), np.sqrt(5 / (64 * np.pi)) * (1 - c) ** 2 * np.exp(-2j * ph), atol=1e-14)
    assert np.allclose(psi4.swsh(-2, 2, 0, th, ph), np.sqrt(15 / (32 * np.pi)) * np.sin(th) ** 2, atol=1e-14)
    _, T, P, W = psi4.sphere_points(1.0, 12, 24)
    lm = [(l, m) for l in range(2, 6) for m in range(-l, l + 1)]
    Ys = {k: psi4.swsh(-2, k[0], k[1], T, P) for k in lm}
    for a in lm:
        for b in lm:
            v = np.sum(W * Ys[a] * np.conj(Ys[b]))
            assert abs(v - (1.0 if a == b else 0.0)) < 1e-12, (a, b, v)


def test_sphere_interpolation_and_mode_recovery():
    cfg = configs.small_bbh(lmax=4, rho=0.4)
    m = OracleMesh(cfg)
    unit = cfg.width / m.L
    ijk = np.stack(np.meshgrid(np.arange(7), np.arange(7), np.arange(7), indexing="ij"), -1)
    ijk = ijk.reshape(-1, 3)[:, ::-1]
    Xn = 6 * m.anchors[:, None, :] + ijk[None] * m.side[:, None, None]
    xn = [cfg.xmin[a] + Xn[..., a] * unit for a in range(3)]
    poly = lambda x, y, z: 1.0 + 0.3 * x ** 6 / 1e6 - 0.2 * y ** 5 * z / 1e6 + x * y * z ** 4 / 1e7
    vals = poly(*xn)                                           # [n_oct, 343]
    xyz, T, P, W = psi4.sphere_points(7.3, 8, 16, center=(0.4, -0.2, 0.1))
    got, _ = psi4.interpolate(m, vals, xyz)
    assert np.max(np.abs(got - poly(*xyz))) < 1e-12 * np.max(np.abs(vals))
    # synthetic Psi_4 from known modes
    rng = np.random.default_rng(3)
    a = {(l, mm): rng.normal() + 1j * rng.normal() for l in range(2, 5) for mm in range(-l, l + 1)}
    field = sum(v * psi4.swsh(-2, l, mm, T, P) for (l, mm), v in a.items())
    got = psi4.modes(field, T, P, W, l_max=4)
    for k, v in a.items():
        assert abs(got[k] - v) < 1e-12
