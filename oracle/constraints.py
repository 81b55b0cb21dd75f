"""ORACLE (test infrastructure only): constraint diagnostics.

Not in the paper (BASELINE.json north_star asks for dgr_constraints); the
standard BSSN forms of SURVEY.md §8c-O9:
    H   = chi gt^ij R_ij + 2/3 K^2 - At_ij At^ij
    M^i = d_j At^ij + Gt^i_jk At^jk - 2/3 gt^ij d_j K - 3/(2 chi) At^ij d_j chi,
          d_j At^ij by the chain rule from d gt and d At
    G^i = Gt^i - gt^jk Gt^i_jk
Output order: H, M^0, M^1, M^2, G^0, G^1, G^2 on the DOFs (zip owners).
"""
from __future__ import annotations

import numpy as np

from .bssn import NF, Params, PointData, geometry
from .maps import OracleMesh
from .rk4 import octant_h
from .unzip import unzip, zip_rhs

NC = 7


def constraints_patches(P, h, prm: Params, chunk=512):
    P = np.asarray(P).reshape(NF, -1, 13, 13, 13)
    n = P.shape[1]
    out = np.empty((NC, n, 7, 7, 7))
    for i0 in range(0, n, chunk):
        i1 = min(n, i0 + chunk)
        out[:, i0:i1] = constraints_point(PointData(P[:, i0:i1], np.asarray(h)[i0:i1]), prm)
    return out


def constraints_point(d, prm: Params):
    """[7, ...] from point data d (values and derivatives, see bssn.PointData)."""
    G = geometry(d, prm)
    ginv, chi = G["ginv"], G["chi"]
    A_up = np.einsum("ik...,jl...,kl...->ij...", ginv, ginv, d.At)
    H = (d.chi * np.einsum("ij...,ij...->...", ginv, G["Ric"])
         + (2.0 / 3.0) * d.K * d.K - np.einsum("ij...,ij...->...", d.At, A_up))
    # d_m gt^ik = -gt^ia d_m gt_ab gt^bk
    d_ginv = -np.einsum("ia...,mab...,bk...->mik...", ginv, d.d_gt, ginv)
    d_Aup = (np.einsum("mik...,jl...,kl...->mij...", d_ginv, ginv, d.At)
             + np.einsum("ik...,mjl...,kl...->mij...", ginv, d_ginv, d.At)
             + np.einsum("ik...,jl...,mkl...->mij...", ginv, ginv, d.d_At))
    M = (np.einsum("jij...->i...", d_Aup)
         + np.einsum("ijk...,jk...->i...", G["Gam"], A_up)
         - (2.0 / 3.0) * np.einsum("ij...,j...->i...", ginv, d.d_K)
         - 1.5 / chi * np.einsum("ij...,j...->i...", A_up, d.d_chi))
    Gc = d.Gt - G["CalGt"]
    return np.concatenate([H[None], M, Gc])


def constraints_dofs(mesh: OracleMesh, u, prm: Params):
    P = unzip(mesh, u)
    c = constraints_patches(P, octant_h(mesh), prm)
    return zip_rhs(mesh, c.reshape(NC, mesh.n_oct, 343))


def norms(c):
    """[NC, 2]: RMS and max-abs of each constraint over the DOFs."""
    return np.stack([np.sqrt(np.mean(c * c, axis=1)), np.max(np.abs(c), axis=1)], axis=1)
