"""Closed-form spacetimes for the RHS and constraint pins (test helper, sympy).

Each solution is written from its ADM data (gamma_ij, alpha, beta^i, K_ij) and
converted to BSSN variables here, independently of synth/ and oracle/:
    chi = det(gamma)^(-1/3), gt_ij = chi gamma_ij, K = gamma^ij K_ij,
    At_ij = chi (K_ij - gamma_ij K / 3), Gt^i = -d_j gt^ij   (det gt = 1).
pointdata() evaluates values and exact first/second derivatives at points in
the layout of oracle.bssn.PointData, so the oracle's algebra can be checked
with no finite differences in the loop.
"""
from types import SimpleNamespace

import numpy as np
import sympy as sp

X, Y, Z, T = sp.symbols("x y z t", real=True)
XYZ = (X, Y, Z)
SYM = [(0, 0), (0, 1), (0, 2), (1, 1), (1, 2), (2, 2)]


def bssn_from_adm(gamma, alpha, beta, Kij, gamma_inv=None):
    det = sp.simplify(gamma.det())
    chi = det ** sp.Rational(-1, 3)
    gt = chi * gamma
    ginv_phys = gamma_inv if gamma_inv is not None else gamma.inv()
    gtinv = ginv_phys / chi
    Ktr = sum(ginv_phys[i, j] * Kij[i, j] for i in range(3) for j in range(3))
    At = chi * (Kij - gamma * Ktr / 3)
    Gt = [-sum(sp.diff(gtinv[i, j], XYZ[j]) for j in range(3)) for i in range(3)]
    f = [alpha, chi, Ktr] + Gt + list(beta) + [0, 0, 0] \
        + [gt[i, j] for (i, j) in SYM] + [At[i, j] for (i, j) in SYM]
    return [sp.sympify(e) for e in f]


def gauge_wave(amp=sp.Rational(1, 10), d=1):
    """Apples-with-Apples gauge wave: ds^2 = -H dt^2 + H dx^2 + dy^2 + dz^2,
    H = 1 - A sin(2 pi (x - t)/d); beta = 0, K_ij = -d_t gamma_ij / (2 alpha)."""
    H = 1 - amp * sp.sin(2 * sp.pi * (X - T) / d)
    gamma = sp.diag(H, 1, 1)
    alpha = sp.sqrt(H)
    Kij = -sp.diff(gamma, T) / (2 * alpha)
    return bssn_from_adm(gamma, alpha, [0, 0, 0], Kij)


def kerr_schild(M=1):
    """Schwarzschild in Kerr-Schild coordinates (closed-form K_ij)."""
    r = sp.sqrt(X ** 2 + Y ** 2 + Z ** 2)
    l = [X / r, Y / r, Z / r]
    H = M / r
    gamma = sp.Matrix(3, 3, lambda i, j: sp.KroneckerDelta(i, j) + 2 * H * l[i] * l[j])
    ginv = sp.Matrix(3, 3, lambda i, j: sp.KroneckerDelta(i, j) - 2 * H / (1 + 2 * H) * l[i] * l[j])
    alpha = 1 / sp.sqrt(1 + 2 * H)
    beta = [2 * H / (1 + 2 * H) * l[i] for i in range(3)]
    Kij = sp.Matrix(3, 3, lambda i, j: 2 * M * alpha / r ** 2
                    * (sp.KroneckerDelta(i, j) - (2 + M / r) * l[i] * l[j]))
    return bssn_from_adm(gamma, alpha, beta, Kij, gamma_inv=ginv), (gamma, ginv)


def _lam(e):
    return sp.lambdify((X, Y, Z, T), e, modules="numpy")


def _ev(e, pts, t=0.0):
    v = _lam(e)(pts[0], pts[1], pts[2], t)
    return np.broadcast_to(np.asarray(v, dtype=np.float64), pts[0].shape).copy()


def pointdata(fields, pts, t=0.0, second=True):
    """fields: 24 sympy expressions in x,y,z(,t); pts: [3, n] numpy."""
    ev = lambda e: _ev(e, pts, t)
    d1 = lambda e: np.stack([ev(sp.diff(e, v)) for v in XYZ])
    d2 = lambda e: np.stack([np.stack([ev(sp.diff(e, a, b)) for b in XYZ]) for a in XYZ])

    def full(vals):
        out = np.empty((3, 3) + vals[0].shape)
        for q, (i, j) in enumerate(SYM):
            out[i, j] = out[j, i] = vals[q]
        return out

    d = SimpleNamespace()
    d.alpha, d.chi, d.K = ev(fields[0]), ev(fields[1]), ev(fields[2])
    d.Gt = np.stack([ev(fields[3 + i]) for i in range(3)])
    d.beta = np.stack([ev(fields[6 + i]) for i in range(3)])
    d.B = np.stack([ev(fields[9 + i]) for i in range(3)])
    d.gt = full([ev(fields[12 + q]) for q in range(6)])
    d.At = full([ev(fields[18 + q]) for q in range(6)])
    d.d_alpha, d.d_chi, d.d_K = d1(fields[0]), d1(fields[1]), d1(fields[2])
    d.d_Gt = np.stack([d1(fields[3 + i]) for i in range(3)], axis=1)
    d.d_beta = np.stack([d1(fields[6 + i]) for i in range(3)], axis=1)
    d.d_B = np.stack([d1(fields[9 + i]) for i in range(3)], axis=1)
    dg = [d1(fields[12 + q]) for q in range(6)]
    d.d_gt = np.stack([full([dg[q][k] for q in range(6)]) for k in range(3)])
    dA = [d1(fields[18 + q]) for q in range(6)]
    d.d_At = np.stack([full([dA[q][k] for q in range(6)]) for k in range(3)])
    if second:
        d.dd_alpha, d.dd_chi = d2(fields[0]), d2(fields[1])
        d.dd_beta = np.stack([d2(fields[6 + i]) for i in range(3)], axis=2)
        ddg = [d2(fields[12 + q]) for q in range(6)]
        d.dd_gt = np.empty((3, 3, 3, 3) + pts[0].shape)
        for k in range(3):
            for l in range(3):
                d.dd_gt[k, l] = full([ddg[q][k, l] for q in range(6)])
    return d


def time_derivative(fields, pts, t=0.0):
    """[24, n] exact d/dt of the BSSN fields (for time-dependent solutions)."""
    return np.stack([_ev(sp.diff(e, T), pts, t) for e in fields])


def values(fields, pts, t=0.0):
    return np.stack([_ev(e, pts, t) for e in fields])
