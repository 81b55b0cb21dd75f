"""ORACLE (test infrastructure only): finite differences on 13^3 patches.

PAPER.md L95 (§III-A): "finite difference stencils that are O(h^6)"; L310
(§IV-B): 72 first derivatives (all 24 fields), 66 second derivatives (all six
second derivatives of alpha, beta^i, chi, gamma~_ij), 72 Kreiss-Oliger terms.
Stencils (readings R8-R10):
    D1 u = ((u1-u-1)*45 - (u2-u-2)*9 + (u3-u-3)) / (60 h)
    D2 u = (2(u3+u-3) - 27(u2+u-2) + 270(u1+u-1) - 490 u0) / (180 h^2)
    D_ab u = D1_a (D1_b u)                          (mixed, tensor product)
    KO_a u = sigma/(64 h) * (u-3 - 6u-2 + 15u-1 - 20u0 + 15u1 - 6u2 + u3)
Patches are indexed [..., z, y, x]; axis a = 0,1,2 means x, y, z.
Outputs are on the 7^3 interior (patch indices 3..9).
"""
from __future__ import annotations

import numpy as np

K, R = 3, 7


def _arr_axis(a: int) -> int:
    return -1 - a          # x -> -1, y -> -2, z -> -3


def _sl(P, a, s, ext=()):
    """View of P shifted by s along axis a; interior (3..9) along every other
    axis except those in `ext` (kept full 0..12)."""
    idx = [slice(None)] * P.ndim
    for b in range(3):
        ax = P.ndim + _arr_axis(b)
        if b == a:
            idx[ax] = slice(K + s, K + s + R)
        elif b in ext:
            idx[ax] = slice(None)
        else:
            idx[ax] = slice(K, K + R)
    return P[tuple(idx)]


def d1(P, a, h, ext=()):
    u = lambda s: _sl(P, a, s, ext)
    return ((u(1) - u(-1)) * 45.0 - (u(2) - u(-2)) * 9.0 + (u(3) - u(-3))) / (60.0 * h)


def d2(P, a, h):
    u = lambda s: _sl(P, a, s)
    return (2.0 * (u(3) + u(-3)) - 27.0 * (u(2) + u(-2)) + 270.0 * (u(1) + u(-1))
            - 490.0 * u(0)) / (180.0 * h * h)


def dmixed(P, a, b, h):
    """D1_a(D1_b u): D1_b is first taken on the 13-wide extent along a."""
    inner = d1(P, b, h, ext=(a,))          # [..., 7 or 13 per axis]: full along a
    # re-embed into a 13^3 frame so _sl can shift along a
    shp = list(P.shape)
    Q = np.zeros(shp)
    idx = [slice(None)] * P.ndim
    for c in range(3):
        ax = P.ndim + _arr_axis(c)
        idx[ax] = slice(None) if c == a else slice(K, K + R)
    Q[tuple(idx)] = inner
    return d1(Q, a, h)


def ko(P, a, h, sigma):
    u = lambda s: _sl(P, a, s)
    return (sigma / (64.0 * h)) * (u(-3) - 6.0 * u(-2) + 15.0 * u(-1) - 20.0 * u(0)
                                   + 15.0 * u(1) - 6.0 * u(2) + u(3))


def lop_plus(P, a, h):
    """4th-order lopsided first derivative shifted towards +a (reading R9u):
    (-3 u-1 - 10 u0 + 18 u1 - 6 u2 + u3) / (12 h)."""
    u = lambda s: _sl(P, a, s)
    return (-3.0 * u(-1) - 10.0 * u(0) + 18.0 * u(1) - 6.0 * u(2) + u(3)) / (12.0 * h)


def lop_minus(P, a, h):
    """Its mirror image, shifted towards -a: (3 u1 + 10 u0 - 18 u-1 + 6 u-2 - u-3) / (12 h)."""
    u = lambda s: _sl(P, a, s)
    return (3.0 * u(1) + 10.0 * u(0) - 18.0 * u(-1) + 6.0 * u(-2) - u(-3)) / (12.0 * h)


def advect(P, beta, h, upwind):
    """beta^k d_k u on the interior: centred D1 (reading R9) or, with upwind,
    the lopsided stencil on the side beta^k points to (beta^k >= 0 -> +k)."""
    out = 0.0
    for a in range(3):
        if upwind:
            d = np.where(beta[a] >= 0.0, lop_plus(P, a, h), lop_minus(P, a, h))
        else:
            d = d1(P, a, h)
        out = out + beta[a] * d
    return out


def interior(P):
    return P[..., K:K + R, K:K + R, K:K + R]


def grad(P, h):
    """[3, ...] first derivatives."""
    return np.stack([d1(P, a, h) for a in range(3)])


def hess(P, h):
    """[3, 3, ...] second derivatives (symmetric; mixed via D1 o D1)."""
    out = np.empty((3, 3) + P.shape[:-3] + (R, R, R))
    for a in range(3):
        out[a, a] = d2(P, a, h)
        for b in range(a + 1, 3):
            out[a, b] = out[b, a] = dmixed(P, a, b, h)
    return out


def ko_sum(P, h, sigma):
    return ko(P, 0, h, sigma) + ko(P, 1, h, sigma) + ko(P, 2, h, sigma)
