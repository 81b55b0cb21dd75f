"""ORACLE (test infrastructure only): Sommerfeld radiative outer boundary.

SURVEY.md §8f item 2.  PAPER.md is silent on the outer boundary (reading R12:
degree-6 extrapolation of the padding); this module adds the radiative
condition as reading R29, applied to the right-hand side at every
DOF that lies on a face of a non-periodic domain:

    d_t f = -(x^i / r) d_i f - (f - f_inf) / r,      r = |x|,

with unit propagation speed and unit fall-off for every field, f_inf = 1 for
alpha, chi and gt_xx, gt_yy, gt_zz and 0 for every other field, x the physical
coordinates (the domains are centred on the origin), and d_i f the same
centred 6th-order first derivative the RHS uses (fd.d1 on the patch, whose
padding is extrapolated outside the domain, R12).  The condition replaces the
whole right-hand side (algebra and KO) at those points.  An outgoing spherical
wave f = f_inf + g(r - t)/r satisfies it exactly (pinned in
tests/test_oracle_boundary.py).
"""
from __future__ import annotations

import numpy as np

from . import fd
from .bssn import F_ALPHA, F_CHI, F_GAM, NF
from .maps import _local_ijk

F_INF = np.zeros(NF)
F_INF[[F_ALPHA, F_CHI, F_GAM + 0, F_GAM + 3, F_GAM + 5]] = 1.0


def sommerfeld_rhs(f, grad, x, f_inf):
    """The radiative condition for values f [...], gradients grad [3, ...] at
    physical points x [3, ...] (r = |x| > 0)."""
    r = np.sqrt(x[0] * x[0] + x[1] * x[1] + x[2] * x[2])
    return -(x[0] * grad[0] + x[1] * grad[1] + x[2] * grad[2]) / r - (f - f_inf) / r


def boundary_points(mesh, octs):
    """[n, 343] bool: interior patch point (= element node) of octant octs[i]
    lies on a face of the (non-periodic) domain; and its lattice coordinates."""
    octs = np.asarray(octs, dtype=np.int64)
    X = mesh.node_X(octs[:, None], _local_ijk()[None, :, :])      # [n, 343, 3]
    on = np.any((X == 0) | (X == mesh.L), axis=2)
    return on, X


def apply_sommerfeld(mesh, octs, P, r):
    """Replace r [24, n, 7, 7, 7] (RHS at the interior points of the patches P
    [24, n, 13, 13, 13] of octants octs) by the radiative condition at every
    point on the outer boundary.  No-op on periodic domains."""
    if mesh.periodic:
        return r
    octs = np.asarray(octs, dtype=np.int64)
    on, X = boundary_points(mesh, octs)
    if not on.any():
        return r
    unit = mesh.cfg.width / mesh.L
    x = np.stack([mesh.cfg.xmin[a] + X[..., a] * unit for a in range(3)])   # [3, n, 343]
    hh = np.asarray([mesh.h(e) for e in octs])[:, None, None, None]
    P = np.asarray(P).reshape(NF, len(octs), 13, 13, 13)
    r = r.reshape(NF, len(octs), 343).copy()
    xs = x[:, on]
    for f in range(NF):
        g = np.stack([fd.d1(P[f], a, hh) for a in range(3)]).reshape(3, len(octs), 343)
        val = fd.interior(P[f]).reshape(len(octs), 343)
        r[f][on] = sommerfeld_rhs(val[on], g[:, on], xs, F_INF[f])
    return r
