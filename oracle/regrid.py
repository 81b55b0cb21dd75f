"""ORACLE (test infrastructure only): regrid — wavelet refinement indicator,
new octree, intergrid transfer (Alg. 1 line 3
`construct_grid(u)`: "the host generates the grid (or re-grids)
and passes the data to the device"; refinement by an error
tolerance epsilon).  The paper delegates all of it to DENDRO-GR
without giving formulas, so this module follows the readings of DESIGN.md §2:

R30 wavelet indicator.  For each octant e and field f, take its 13^3 patch P
    (the unzip of Alg. 2).  The patch points with all-even indices
    (0, 2, .., 12 per axis) form a grid of spacing 2h around e; predict every
    interior point (indices 3..9) from it by the tensor degree-6 Lagrange
    interpolant (the 13x7 table of: along an axis with even index the
    point is a grid point, along an odd one the 7-point row l_m(i/2)).  The
    wavelet coefficient is |P - prediction|; w_e is its maximum over the
    interior points and the selected fields.  (Exactly 0 at the all-even
    points; 0 up to rounding for data that are polynomials of degree <= 6 per
    axis.)
R31 new octree.  A leaf with w_e > eps_refine and level < level_max is split
    into its 8 children; a complete family of 8 sibling leaves, none split,
    all with w_e < eps_coarsen and level > level_min, is merged into its
    parent; then the minimal 2:1 vertex-balance closure (octree.balance) and
    Morton order.  Every leaf changes by at most one level.
R32 transfer.  The value at a DOF X of the new mesh is the old mesh's
    piecewise interpolant at X: the degree-6 tensor Lagrange interpolant of
    the finest old leaf whose closed box contains X (lowest Morton index on
    ties), with that leaf's hanging nodes reconstructed (Alg. 2 l.4-5).  With
    levels changing by at most one, X is on the half-grid of that leaf (the
    same 13x7 table).
"""
from __future__ import annotations

import numpy as np

from .maps import R, OracleMesh
from .octree import balance, children, sort_morton
from .unzip import W13, _interp_points, _t2, elements, unzip


def _pred_rows():
    """[7, 7]: row r (interior patch index 3 + r) over the even points m
    (patch index 2m): a unit vector at even index, W13[index] at odd."""
    rows = np.zeros((R, R))
    for r in range(R):
        i = 3 + r
        if i % 2 == 0:
            rows[r, i // 2] = 1.0
        else:
            rows[r] = W13[i]
    return rows


def wavelet_indicator(mesh: OracleMesh, u: np.ndarray, fields=None, chunk=2000):
    """w [n_oct] (reading R30)."""
    fields = list(range(u.shape[0])) if fields is None else list(fields)
    Rw = _pred_rows()
    w = np.zeros(mesh.n_oct)
    for o0 in range(0, mesh.n_oct, chunk):
        octs = np.arange(o0, min(mesh.n_oct, o0 + chunk))
        P = unzip(mesh, u[fields], octs)                       # [nf, n, z, y, x]
        Pe = P[:, :, ::2, ::2, ::2]                            # even points [.., 7, 7, 7]
        pred = np.einsum("kc,jb,ia,fncba->fnkji", Rw, Rw, Rw, Pe, optimize=True)
        coef = np.abs(P[:, :, 3:10, 3:10, 3:10] - pred)
        w[octs] = coef.max(axis=(0, 2, 3, 4))
    return w


def new_octree(mesh: OracleMesh, w, eps_refine, eps_coarsen, level_min, level_max):
    """(anchors, levels) of the regridded octree (reading R31)."""
    a, l = mesh.anchors, mesh.levels
    D = mesh.D
    refine = (w > eps_refine) & (l < level_max)
    # complete families of leaf siblings: same parent, 8 leaves of the same level
    side = np.int64(1) << (D - l)
    parent = a & ~(2 * side[:, None] - 1)                      # anchor of the parent
    key = {}
    for e in range(mesh.n_oct):
        if l[e] == 0:
            continue
        key.setdefault((l[e], *parent[e]), []).append(e)
    merge = np.zeros(mesh.n_oct, dtype=bool)
    par_a, par_l = [], []
    for (lv, *pa), fam in key.items():
        if (len(fam) == 8 and lv > level_min and not refine[fam].any()
                and np.all(w[fam] < eps_coarsen)):
            merge[fam] = True
            par_a.append(pa)
            par_l.append(lv - 1)
    keep = ~refine & ~merge
    ca, cl = children(a[refine], l[refine], D)
    na = np.concatenate([a[keep], ca, np.array(par_a, dtype=np.int64).reshape(-1, 3)])
    nl = np.concatenate([l[keep], cl, np.array(par_l, dtype=np.int64)])
    na, nl = sort_morton(na, nl, D)
    return balance(na, nl, D, mesh.periodic)


def transfer(old: OracleMesh, u_old: np.ndarray, new: OracleMesh, chunk=20000):
    """u_new [nf, new.n_dof] (reading R32)."""
    new.build_dofs()
    E = elements(old, u_old)
    X = new.dof_lattice()
    out = np.empty((u_old.shape[0], len(X)))
    for i0 in range(0, len(X), chunk):
        Xc = X[i0:i0 + chunk]
        cand = old.containing(Xc)                              # [M, 8]
        lv = np.where(cand >= 0, old.levels[np.maximum(cand, 0)], -1)
        best = lv.max(axis=1)
        # finest containing leaf, lowest Morton index among them
        big = np.iinfo(np.int64).max
        c = np.where(lv == best[:, None], cand, big).min(axis=1)
        t2 = _t2(old, Xc, c)
        out[:, i0:i0 + len(Xc)] = _interp_points(E, c, t2)
    return out
