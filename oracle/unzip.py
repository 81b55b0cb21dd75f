"""ORACLE (test infrastructure only): octant-to-patch ("unzip") and
patch-to-octant ("zip").

PAPER.md Alg. 2 (L249-283) and §IV-A (L235-306): every octant's 7^3 nodal
values are loaded (u[O2N[e]]), hanging values are reconstructed by
interpolation from the coarser neighbour (interp_hanging, L261-264), then the
padding zone of each patch is filled by a direct copy (same level), injection
(source finer) or interpolation (source coarser) — "tensor products of 1D
interpolation operators" (L295).  Patch-to-octant copies the interior points
back (L297).

The oracle evaluates every value from its definition:
    value(x) = I_src(x) = sum_{i,j,k} l_i(tx) l_j(ty) l_k(tz) E_src[i,j,k],
with l_m the degree-6 Lagrange basis on the nodes t = 0..6 of the source
octant; points outside a non-periodic domain are filled afterwards by degree-6
polynomial extrapolation along x, then y, then z (reading R12).
"""
from __future__ import annotations

from fractions import Fraction

import numpy as np

from .maps import (K, KIND_COPY, KIND_EXTRAP, KIND_INJECT, KIND_INTERP, KIND_SELF,
                   KIND_WRAP, P13, R, OracleMesh, _local_ijk, _patch_ijk)


def lagrange_weights(t: Fraction):
    """l_m(t), m = 0..6, for the degree-6 Lagrange basis on nodes 0..6 (exact rationals)."""
    w = []
    for m in range(R):
        v = Fraction(1)
        for q in range(R):
            if q != m:
                v *= Fraction(t - q, m - q)
        w.append(v)
    return w


def interp_table():
    """13 x 7 table: row t2 holds l_m(t2/2) (dyadic rationals -> exact in fp64)."""
    return np.array([[float(x) for x in lagrange_weights(Fraction(t2, 2))] for t2 in range(13)])


def extrap_rows():
    """Rows for t = -1, -2, -3 (integers): extrapolation below node 0."""
    return np.array([[float(x) for x in lagrange_weights(Fraction(-t))] for t in (1, 2, 3)])


W13 = interp_table()
WEXT = extrap_rows()


def _interp_points(E, c, t2):
    """I_c at half-integer coordinates t2 ([M,3] ints in 0..12) for sources c ([M]):
        sum_{i,j,k} W13[t2x][i] W13[t2y][j] W13[t2z][k] E_c[i + 7j + 49k].
    Rows W13[t2] with even t2 are unit vectors, so along such an axis the sum
    has the single term of node t2/2; the terms dropped are exact zeros.
    Points are grouped by which axes are odd (8 patterns) only to keep the
    gathers small.  E: [nf, n_oct, 343].  Returns [nf, M]."""
    nf = E.shape[0]
    out = np.empty((nf, len(c)))
    odd = (t2 % 2 == 1)
    pat = odd[:, 0] * 1 + odd[:, 1] * 2 + odd[:, 2] * 4
    ar = np.arange(R)
    for p in range(8):
        sel = np.nonzero(pat == p)[0]
        if len(sel) == 0:
            continue
        idx, wts = [], []
        for a in range(3):
            t = t2[sel, a]
            if (p >> a) & 1:
                idx.append(np.broadcast_to(ar, (len(sel), R)))
                wts.append(W13[t])
            else:
                idx.append((t // 2)[:, None])
                wts.append(np.ones((len(sel), 1)))
        n = (idx[0][:, None, None, :] + R * idx[1][:, None, :, None]
             + R * R * idx[2][:, :, None, None])                         # [m, z, y, x]
        vals = E[:, c[sel][:, None, None, None], n]                     # [f, m, z, y, x]
        out[:, sel] = np.einsum("fmzyx,mx,my,mz->fm", vals, wts[0], wts[1], wts[2],
                                optimize=True)
    return out


def _t2(mesh: OracleMesh, X, c):
    off = mesh._offset(X, c)
    num = 2 * off
    s = mesh.side[c][:, None]
    assert np.all(num % s == 0), "point not on the half-grid of its source"
    t2 = num // s
    assert np.all((t2 >= 0) & (t2 <= 12))
    return t2


def elements(mesh: OracleMesh, u: np.ndarray, chunk=20000) -> np.ndarray:
    """E [nf, n_oct, 343]: nodal values of every octant with hanging points
    reconstructed (Alg. 2 lines 2-5), resolved level by level, coarse to fine,
    so chains of hanging points are handled (reading R14)."""
    mesh.build_dofs()
    nf = u.shape[0]
    o2n = mesh.o2n
    E = np.where(o2n[None] >= 0, u[:, np.maximum(o2n, 0)], np.nan)
    ht = mesh.hanging_table()
    if len(ht):
        ijk = _local_ijk()
        lv = mesh.levels[ht[:, 0]]
        for L in np.unique(lv):
            rows = ht[lv == L]
            for r0 in range(0, len(rows), chunk):
                rr = rows[r0:r0 + chunk]
                X = mesh.node_X(rr[:, 0], ijk[rr[:, 1]])
                t2 = _t2(mesh, X, rr[:, 2])
                vals = _interp_points(E, rr[:, 2], t2)
                assert np.all(np.isfinite(vals)), "hanging chain not resolved in level order"
                E[:, rr[:, 0], rr[:, 1]] = vals
    return E


def unzip(mesh: OracleMesh, u: np.ndarray, octs=None, chunk=4000) -> np.ndarray:
    """Patches [nf, n, 13, 13, 13] (index [z][y][x]) of octants `octs` (default all)."""
    return unzip_from_elements(mesh, elements(mesh, u), octs, chunk)


def padding_sources_cached(mesh: OracleMesh, octs):
    """mesh.padding_sources(octs), memoised for the whole mesh (the maps do not depend on u)."""
    if getattr(mesh, "_pad_cache", None) is None:
        mesh._pad_cache = mesh.padding_sources()
    src, kind = mesh._pad_cache
    return src[octs], kind[octs]


def unzip_from_elements(mesh: OracleMesh, E: np.ndarray, octs=None, chunk=4000) -> np.ndarray:
    """Octant-to-patch given the reconstructed element values E [nf, n_oct, 343]."""
    full = octs is None
    octs = np.arange(mesh.n_oct) if octs is None else np.asarray(octs, dtype=np.int64)
    nf = E.shape[0]
    if full or getattr(mesh, "_pad_cache", None) is not None:
        src, kind = padding_sources_cached(mesh, octs)
    else:
        src, kind = mesh.padding_sources(octs)
    pijk = _patch_ijk()
    out = np.empty((nf, len(octs), P13 ** 3))
    for i0 in range(0, len(octs), chunk // 8 + 1):
        i1 = min(len(octs), i0 + chunk // 8 + 1)
        ob = octs[i0:i1]
        sv = src[i0:i1].reshape(-1)
        kv = kind[i0:i1].reshape(-1)
        bb = np.repeat(ob, P13 ** 3)
        X = 6 * mesh.anchors[bb] + (np.tile(pijk, (len(ob), 1)) - K) * mesh.side[bb][:, None]
        vals = np.full((nf, len(bb)), np.nan)
        ok = (kv & 7) != KIND_EXTRAP
        idx = np.nonzero(ok)[0]
        for j0 in range(0, len(idx), 200000):
            jj = idx[j0:j0 + 200000]
            c = sv[jj]
            t2 = _t2(mesh, X[jj], c)
            vals[:, jj] = _interp_points(E, c, t2)
        out[:, i0:i1, :] = vals.reshape(nf, len(ob), -1)
    P = out.reshape(nf, len(octs), P13, P13, P13)
    if not mesh.periodic:
        _extrapolate(mesh, P, octs)
    assert np.all(np.isfinite(P))
    return P


def _extrapolate(mesh: OracleMesh, P, octs):
    """Phase B (reading R12): for a = x, y, z in order, every patch point that
    is outside the domain along a and inside along all later axes is the
    degree-6 polynomial through patch indices 3..9 along a, evaluated at
    t = -1,-2,-3 (indices 2,1,0) or, mirrored, at indices 10,11,12."""
    pr = np.arange(P13)
    for a in range(3):   # 0 = x (last array axis), 1 = y, 2 = z
        # coordinate of patch index i along axis ax for every octant
        def outside(ax):
            X = 6 * mesh.anchors[octs, ax][:, None] + (pr[None, :] - K) * mesh.side[octs][:, None]
            return (X < 0) | (X > mesh.L)                       # [n, 13]
        out_a = outside(a)
        later = [outside(b) for b in range(a + 1, 3)]
        # broadcast masks to [n, z, y, x]
        def bc(m, ax):
            shp = [m.shape[0], 1, 1, 1]
            shp[3 - ax] = P13
            return m.reshape(shp)
        mask = bc(out_a, a)
        for b, mb in zip(range(a + 1, 3), later):
            mask = mask & ~bc(mb, b)
        arr_ax = 4 - a                                            # axis in P[f, n, z, y, x]
        Pm = np.moveaxis(P, arr_ax, -1)                           # [..., 13] along a
        inner = Pm[..., K:K + R]
        ext = np.empty(Pm.shape[:-1] + (P13,))
        for t in range(3):                                        # t=-1,-2,-3
            ext[..., K - 1 - t] = inner @ WEXT[t]
            ext[..., K + R + t] = inner[..., ::-1] @ WEXT[t]
        ext[..., K:K + R] = inner
        mk = np.moveaxis(np.broadcast_to(mask, P.shape[1:]), arr_ax - 1, -1)
        Pm[..., :] = np.where(mk[None], ext, Pm)
        P[...] = np.moveaxis(Pm, -1, arr_ax)


def zip_rhs(mesh: OracleMesh, rhs_oct: np.ndarray) -> np.ndarray:
    """Patch-to-octant: DOF value = the owner octant's interior value
    (zip owner: coarsest containing leaf, lowest index; reading R17).
    rhs_oct: [nf, n_oct, 343] -> [nf, n_dof]."""
    mesh.build_dofs()
    return rhs_oct[:, mesh.zip_leaf, mesh.zip_node]
