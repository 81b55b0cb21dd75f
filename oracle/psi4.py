"""ORACLE (test infrastructure only): gravitational-wave extraction — the
Weyl scalar Psi_4 on the octree, interpolated to extraction spheres and
projected on spin-weight -2 spherical harmonics (the
other half of "regrid or Psi_4").

PAPER.md P:L159: "We use the Penrose scalar Psi_4 [37], [44] for gravitational
wave extraction ... expanding it in a basis of spin-weighted spherical
harmonics (l, m modes) on spherical shells; integrations being performed
using Lebedev quadrature [45]."  The paper gives no formula; the readings
 are the standard 3+1 forms of its reference [44] (Bishop &
Rezzolla):

R33  Psi_4 = (E_ij - i B_ij) mbar^i mbar^j with, in vacuum,
       E_ij = R_ij + K K_ij - K_ik gamma^kl K_lj,
       B_ij = 1/2 (eps_i^kl D_k K_lj + eps_j^kl D_k K_li),
     gamma_ij = gt_ij / chi, K_ij = (At_ij + gt_ij K / 3) / chi, R_ij the Ricci
     tensor of gamma (eqs 16-19, oracle.bssn.geometry), D_k the covariant
     derivative of gamma (Christoffels of eq 13), eps^ijk = [ijk] / sqrt(gamma),
     eps_i^kl = gamma_im eps^mkl.
R34  tetrad: the coordinate directions r^ = x/r, theta^ = (xz, yz, -(x^2 +
     y^2)) / (r rho), phi^ = (-y, x, 0) / rho about the extraction centre
     (rho = sqrt(x^2 + y^2)), Gram-Schmidt orthonormalised in gamma in that
     order; m = (e_theta + i e_phi) / sqrt(2).  (On flat, linearised data an
     outgoing wave h_+, h_x then has Psi_4 = -h''_+ + i h''_x.)
R35  quadrature: Gauss-Legendre in cos(theta) x uniform in phi (exact for
     spherical harmonics of degree < 2 n_theta and |m| < n_phi) in place of
     Lebedev's rules, whose node tables are not in the paper.
R36  Psi_4 at a sphere point: the degree-6 tensor Lagrange interpolant of its
     values at the 343 nodes of the finest octant containing the point (lowest
     Morton index on ties), each octant evaluating Psi_4 at its own nodes from
     its own patch.
     Spin-weighted harmonics: Goldberg et al. (1967), -2Y_22 = sqrt(5/(64 pi))
     (1 + cos theta)^2 e^{2 i phi}.
"""
from __future__ import annotations

from math import comb, factorial, pi, sqrt

import numpy as np

from .bssn import Params, PointData, geometry
from .maps import OracleMesh
from .rk4 import octant_h
from .unzip import unzip

PERM = np.zeros((3, 3, 3))
for (i, j, k), sgn in {(0, 1, 2): 1, (1, 2, 0): 1, (2, 0, 1): 1,
                       (0, 2, 1): -1, (2, 1, 0): -1, (1, 0, 2): -1}.items():
    PERM[i, j, k] = sgn


def tetrad(xyz, gamma):
    """Unit e_r, e_theta, e_phi [3, n] (reading R34); gamma [3, 3, n]."""
    x, y, z = xyz
    r = np.sqrt(x * x + y * y + z * z)
    rho = np.sqrt(x * x + y * y)
    v = [np.stack([x, y, z]) / r,
         np.stack([x * z, y * z, -(x * x + y * y)]) / (r * rho),
         np.stack([-y, x, np.zeros_like(x)]) / rho]
    dot = lambda a, b: np.einsum("i...,ij...,j...->...", a, gamma, b)
    e = []
    for w in v:
        for u in e:
            w = w - dot(u, w) * u
        e.append(w / np.sqrt(dot(w, w)))
    return e


def psi4_point(d, xyz, prm: Params = Params()):
    """Psi_4 (complex [n]) from point data d (bssn.PointData layout) at
    positions xyz [3, n] relative to the extraction centre (R33, R34)."""
    G = geometry(d, prm)
    chi = G["chi"]                    # chi_e = max(chi, chi_floor) in divisions (R13)
    gam = d.gt / chi
    gam_inv = chi * G["ginv"]         # (chi_e: gamma = gt / chi_e consistently)
    Kij = (d.At + d.gt * d.K / 3.0) / chi
    # d_k K_ij by the product rule from d At, d gt, d K, d chi
    dK = ((d.d_At + d.d_gt * d.K / 3.0 + np.einsum("ij...,k...->kij...", d.gt, d.d_K) / 3.0) / chi
          - np.einsum("ij...,k...->kij...", d.At + d.gt * d.K / 3.0, d.d_chi) / (chi * chi))
    Gp = G["Gphys"]                                                       # Gamma^m_kl
    DK = (dK - np.einsum("mkl...,mj...->klj...", Gp, Kij)
          - np.einsum("mkj...,lm...->klj...", Gp, Kij))                   # D_k K_lj
    trK = np.einsum("ij...,ij...->...", gam_inv, Kij)
    E = G["Ric"] + trK * Kij - np.einsum("ik...,kl...,lj...->ij...", Kij, gam_inv, Kij)
    sqg = np.sqrt(np.linalg.det(np.moveaxis(gam, (0, 1), (-2, -1))))
    eps_up = PERM.reshape((3, 3, 3) + (1,) * sqg.ndim) / sqg              # eps^{mkl}
    eps_mix = np.einsum("im...,mkl...->ikl...", gam, eps_up)              # eps_i^{kl}
    Bh = np.einsum("ikl...,klj...->ij...", eps_mix, DK)
    B = 0.5 * (Bh + np.einsum("ij...->ji...", Bh))
    _, et, ep = tetrad(xyz, gam)
    mb = (et - 1j * ep) / sqrt(2.0)
    return np.einsum("i...,ij...,j...->...", mb, E - 1j * B, mb)


def psi4_octants(mesh: OracleMesh, u, center=(0.0, 0.0, 0.0), prm: Params = Params(),
                 chunk=512):
    """Psi_4 at the 343 nodes of every octant, from its own patch: [n_oct, 343] complex
    (node n = i + 7 j + 49 k, x fastest)."""
    out = np.empty((mesh.n_oct, 343), dtype=complex)
    h = octant_h(mesh)
    unit = mesh.cfg.width / mesh.L
    ijk = np.stack(np.meshgrid(np.arange(7), np.arange(7), np.arange(7), indexing="ij"), -1)
    ijk = ijk.reshape(-1, 3)[:, ::-1]          # rows in (z, y, x) order -> columns x, y, z
    for o0 in range(0, mesh.n_oct, chunk):
        octs = np.arange(o0, min(mesh.n_oct, o0 + chunk))
        P = unzip(mesh, u, octs)
        d = PointData(P, h[octs])
        X = (6 * mesh.anchors[octs][:, None, :] + ijk[None] * mesh.side[octs][:, None, None])
        xyz = np.stack([mesh.cfg.xmin[a] + X[..., a] * unit - center[a] for a in range(3)])
        xyz = xyz.reshape(3, len(octs), 7, 7, 7)          # [a, e, z, y, x]
        out[octs] = psi4_point(d, xyz, prm).reshape(len(octs), 343)
    return out


def lagrange_float(t):
    """l_m(t), m = 0..6 for real t (nodes 0..6), [7, n]."""
    t = np.asarray(t, dtype=np.float64)
    w = np.ones((7,) + t.shape)
    for m in range(7):
        for q in range(7):
            if q != m:
                w[m] = w[m] * (t - q) / (m - q)
    return w


def sphere_points(radius, n_theta, n_phi, center=(0.0, 0.0, 0.0)):
    """(xyz [3, n], theta [n], phi [n], weights [n]) of the product rule (R35)."""
    x, wx = np.polynomial.legendre.leggauss(n_theta)
    th = np.arccos(x)
    ph = 2.0 * pi * np.arange(n_phi) / n_phi
    TH, PH = np.meshgrid(th, ph, indexing="ij")
    W = np.repeat(wx[:, None], n_phi, axis=1) * (2.0 * pi / n_phi)
    xyz = np.stack([radius * np.sin(TH) * np.cos(PH) + center[0],
                    radius * np.sin(TH) * np.sin(PH) + center[1],
                    radius * np.cos(TH) + center[2]])
    return xyz.reshape(3, -1), TH.ravel(), PH.ravel(), W.ravel()


def containing_leaf(mesh: OracleMesh, X):
    """Finest leaf whose closed box contains the lattice-unit points X [n, 3]
    (float), lowest Morton index on ties (R36): the leaves of the depth-D
    cells around X — one cell per axis, two where X lies on a cell face."""
    cell = X / 6.0
    lo = np.floor(cell).astype(np.int64)
    on = (lo * 6.0 == X)
    best_l = np.full(len(X), -1, dtype=np.int64)
    best_c = np.full(len(X), np.iinfo(np.int64).max, dtype=np.int64)
    for q in range(8):
        c = [np.where(on[:, a] & bool((q >> a) & 1), lo[:, a] - 1, lo[:, a]) for a in range(3)]
        leaf = mesh.loc.leaf_of_cell(c[0], c[1], c[2])
        ok = leaf >= 0
        lv = np.where(ok, mesh.levels[np.maximum(leaf, 0)], -1)
        better = ok & ((lv > best_l) | ((lv == best_l) & (leaf < best_c)))
        best_l = np.where(better, lv, best_l)
        best_c = np.where(better, leaf, best_c)
    return best_c


def interpolate(mesh: OracleMesh, values, xyz):
    """Per-octant nodal values [n_oct, 343] at physical points xyz [3, n] (R36)."""
    unit = mesh.cfg.width / mesh.L
    X = np.stack([(xyz[a] - mesh.cfg.xmin[a]) / unit for a in range(3)], 1)    # lattice units
    c = containing_leaf(mesh, X)
    t = (X - 6.0 * mesh.anchors[c]) / mesh.side[c][:, None]                     # in [0, 6]
    wx, wy, wz = lagrange_float(t[:, 0]), lagrange_float(t[:, 1]), lagrange_float(t[:, 2])
    V = values[c].reshape(-1, 7, 7, 7)                                         # [n, z, y, x]
    return np.einsum("nzyx,xn,yn,zn->n", V, wx, wy, wz), c


def swsh(s, l, m, theta, phi):
    """Spin-weighted spherical harmonic sY_lm (Goldberg et al. 1967)."""
    if l < abs(s) or l < abs(m):
        return np.zeros_like(theta, dtype=complex)
    pre = (-1.0) ** m * sqrt((2 * l + 1) / (4 * pi) * factorial(l + m) * factorial(l - m)
                             / (factorial(l + s) * factorial(l - s)))
    tot = np.zeros_like(theta, dtype=float)
    for r in range(0, l - s + 1):
        k = r + s - m
        if k < 0 or k > l + s:
            continue
        tot = tot + (comb(l - s, r) * comb(l + s, k) * (-1.0) ** (l - r - s)
                     * np.cos(theta / 2.0) ** (2 * r + s - m) * np.sin(theta / 2.0) ** (2 * l - 2 * r - s + m))
    return pre * tot * np.exp(1j * m * phi)


def modes(psi_on_sphere, theta, phi, weights, l_max=4, s=-2):
    """{(l, m): C_lm = sum_q w_q Psi_4(q) conj(sY_lm(q))}, l = 2..l_max."""
    out = {}
    for l in range(abs(s), l_max + 1):
        for m in range(-l, l + 1):
            out[(l, m)] = np.sum(weights * psi_on_sphere * np.conj(swsh(s, l, m, theta, phi)))
    return out
