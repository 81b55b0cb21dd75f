"""ORACLE (test infrastructure only): the 24-field BSSN right-hand side.

Transcribed by hand from PAPER.md §III-A eqs (1)-(19), L97-157, with the
readings of DESIGN.md §Readings:
  R1  eq (17) first term is -1/2 (printed +1/2);
  R2  eq (19) bracket: the -CalGt^m d_m chi term sits inside gt_ij/(2 chi)[...];
  R3  eq (13) "2 gamma" is 2 chi;
  R4  eq (8) is taken from L117-119 (L115 is a truncated duplicate);
  R5  Lie-derivative weights: w = -2/3 for gt_ij and At_ij, 0 for scalars;
  R6  f(alpha) = lambda_f0 + lambda_f1*alpha (default 1), eta = 2;
  R7  undifferentiated Gt^i in (8) and (17) is CalGt^i = gt^jk Gt^i_jk;
  R13 chi in every division is max(chi, chi_floor);
  R9u (Params.upwind = 1, for long moving-puncture runs): every advective
      derivative beta^k d_k f uses the 4th-order lopsided stencil on the side
      beta^k points to (oracle/fd.py lop_plus / lop_minus) instead of the
      centred D1 of R9;
  and the Kreiss-Oliger term (R8) is added to every field after the algebra.
d_t Gt^i in eq (3) is the value of eq (8) before KO is added.

Field order: 0 alpha, 1 chi, 2 K, 3-5 Gt^i, 6-8 beta^i,
9-11 B^i, 12-17 gt_ij, 18-23 At_ij with ij in (xx, xy, xz, yy, yz, zz).
Arrays carry tensor indices first and points last; einsum does the sums.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from . import fd

SYM = [(0, 0), (0, 1), (0, 2), (1, 1), (1, 2), (2, 2)]
F_ALPHA, F_CHI, F_K, F_GT, F_BETA, F_B, F_GAM, F_AT = 0, 1, 2, 3, 6, 9, 12, 18
NF = 24


@dataclass
class Params:
    ko_sigma: float = 0.4
    eta: float = 2.0
    lambda_f0: float = 1.0
    lambda_f1: float = 0.0
    chi_floor: float = 1e-4
    sommerfeld: int = 0        # 1: radiative outer boundary (oracle/boundary.py, R29)
    upwind: int = 0            # 1: lopsided advective derivatives (R9u)


def sym_to_full(v):
    """[6, ...] -> [3, 3, ...]"""
    out = np.empty((3, 3) + v.shape[1:])
    for q, (i, j) in enumerate(SYM):
        out[i, j] = out[j, i] = v[q]
    return out


def full_to_sym(t):
    return np.stack([t[i, j] for (i, j) in SYM])


class PointData:
    """Values and FD derivatives of all fields at the interior points of a set
    of patches.  P: [24, n, 13, 13, 13]; h: [n]."""

    def __init__(self, P, h, upwind=False):
        hh = np.asarray(h, dtype=np.float64)[:, None, None, None]
        I = fd.interior
        self.alpha = I(P[F_ALPHA])
        self.chi = I(P[F_CHI])
        self.K = I(P[F_K])
        self.Gt = np.stack([I(P[F_GT + i]) for i in range(3)])
        self.beta = np.stack([I(P[F_BETA + i]) for i in range(3)])
        self.B = np.stack([I(P[F_B + i]) for i in range(3)])
        self.gt = sym_to_full(np.stack([I(P[F_GAM + q]) for q in range(6)]))
        self.At = sym_to_full(np.stack([I(P[F_AT + q]) for q in range(6)]))
        g = lambda f: fd.grad(P[f], hh)                     # [3(k), ...]
        self.d_alpha = g(F_ALPHA)
        self.d_chi = g(F_CHI)
        self.d_K = g(F_K)
        self.d_Gt = np.stack([g(F_GT + i) for i in range(3)], axis=1)      # [k, i]
        self.d_beta = np.stack([g(F_BETA + i) for i in range(3)], axis=1)  # [k, i]
        self.d_B = np.stack([g(F_B + i) for i in range(3)], axis=1)        # [k, i]
        dg = np.stack([g(F_GAM + q) for q in range(6)], axis=1)           # [k, q]
        self.d_gt = np.stack([sym_to_full(dg[k]) for k in range(3)])       # [k, i, j]
        dA = np.stack([g(F_AT + q) for q in range(6)], axis=1)
        self.d_At = np.stack([sym_to_full(dA[k]) for k in range(3)])       # [k, i, j]
        H = lambda f: fd.hess(P[f], hh)                     # [k, l, ...]
        self.dd_alpha = H(F_ALPHA)
        self.dd_chi = H(F_CHI)
        self.dd_beta = np.stack([H(F_BETA + i) for i in range(3)], axis=2)  # [k, l, i]
        ddg = np.stack([H(F_GAM + q) for q in range(6)], axis=2)           # [k, l, q]
        self.dd_gt = np.empty((3, 3, 3, 3) + ddg.shape[3:])
        for k in range(3):
            for l in range(3):
                self.dd_gt[k, l] = sym_to_full(ddg[k, l])                  # [k, l, i, j]
        # R9u: lopsided advective derivatives beta^k d_k f of every field
        if upwind:
            self.adv = np.stack([fd.advect(P[f], self.beta, hh, True) for f in range(NF)])


def geometry(d: PointData, prm: Params):
    """Inverse metric, Christoffels, Ricci tensor pieces (eqs 12-19)."""
    pts = d.alpha.shape
    # gt^ij: library inverse (np.linalg.inv), points batched
    g = np.moveaxis(d.gt.reshape(3, 3, -1), -1, 0)
    ginv = np.moveaxis(np.linalg.inv(g), 0, -1).reshape((3, 3) + pts)
    chi = np.maximum(d.chi, prm.chi_floor)                  # R13: divisions only
    # first kind Gt_kij = 1/2 (d_i gt_kj + d_j gt_ki - d_k gt_ij)
    C = 0.5 * (np.einsum("ikj...->kij...", d.d_gt) + np.einsum("jki...->kij...", d.d_gt)
               - d.d_gt)
    Gam = np.einsum("kl...,lij...->kij...", ginv, C)        # eq (12)
    CalGt = np.einsum("ij...,kij...->k...", ginv, Gam)
    delta = np.eye(3)
    # eq (13) physical Christoffel (reading R3: 1/(2 chi))
    Gphys = Gam - (np.einsum("ki,j...->kij...", delta, d.d_chi)
                   + np.einsum("kj,i...->kij...", delta, d.d_chi)
                   - np.einsum("ij...,kl...,l...->kij...", d.gt, ginv, d.d_chi)) / (2.0 * chi)
    # eq (15) D_i D_j alpha, eq (14) D^i D_i alpha = chi gt^ij D_i D_j alpha
    DDa = d.dd_alpha - np.einsum("kij...,k...->ij...", Gphys, d.d_alpha)
    DDa_tr = d.chi * np.einsum("ij...,ij...->...", ginv, DDa)
    # eq (17) with reading R1 (-1/2 on the first term); Gt_ijk = gt_il Gt^l_jk
    Gl = np.einsum("il...,ljk...->ijk...", d.gt, Gam)
    Rt = (-0.5 * np.einsum("lm...,lmij...->ij...", ginv, d.dd_gt)
          + 0.5 * (np.einsum("ki...,jk...->ij...", d.gt, d.d_Gt)
                   + np.einsum("kj...,ik...->ij...", d.gt, d.d_Gt))
          + 0.5 * np.einsum("k...,ijk...->ij...", CalGt, Gl + np.einsum("jik...->ijk...", Gl))
          + np.einsum("lm...,kli...,jkm...->ij...", ginv, Gam, Gl)
          + np.einsum("lm...,klj...,ikm...->ij...", ginv, Gam, Gl)
          + np.einsum("lm...,kim...,klj...->ij...", ginv, Gam, Gl))
    # eqs (18)-(19) with reading R2
    Rchi = ((d.dd_chi - np.einsum("kij...,k...->ij...", Gam, d.d_chi)) / (2.0 * chi)
            - np.einsum("i...,j...->ij...", d.d_chi, d.d_chi) / (4.0 * chi * chi)
            + d.gt / (2.0 * chi) * (
                np.einsum("kl...,kl...->...", ginv, d.dd_chi)
                - 1.5 / chi * np.einsum("kl...,k...,l...->...", ginv, d.d_chi, d.d_chi)
                - np.einsum("m...,m...->...", CalGt, d.d_chi)))
    return dict(ginv=ginv, chi=chi, C=C, Gam=Gam, CalGt=CalGt, Gphys=Gphys,
                DDa=DDa, DDa_tr=DDa_tr, Rt=Rt, Rchi=Rchi, Ric=Rt + Rchi)


def algebra(d: PointData, prm: Params):
    """The algebraic part A of the RHS (eqs 1-8) without KO.  Returns [24, ...]."""
    G = geometry(d, prm)
    ginv, chi, Gam, CalGt = G["ginv"], G["chi"], G["Gam"], G["CalGt"]
    a, K = d.alpha, d.K
    div_beta = np.einsum("kk...->...", d.d_beta)

    def adv(f, grad_):
        """beta^k d_k of field f: centred (R9) from its gradient, or lopsided (R9u)"""
        if prm.upwind:
            return d.adv[f]
        return np.einsum("k...,k...->...", d.beta, grad_)

    # eq (10) Lie derivative, weight w = -2/3 (reading R5); f0: field of T_xx
    def lie(T, dT, f0):
        bdT = np.stack([adv(f0 + q, dT[:, i, j]) for q, (i, j) in enumerate(SYM)])
        return (sym_to_full(bdT)
                + np.einsum("ik...,jk...->ij...", T, d.d_beta)
                + np.einsum("kj...,ik...->ij...", T, d.d_beta)
                - (2.0 / 3.0) * T * div_beta)
    def tf(T):                                               # eq (11)
        tr = np.einsum("lm...,lm...->...", ginv, T)
        return T - d.gt * tr / 3.0
    A_up = np.einsum("ik...,jl...,kl...->ij...", ginv, ginv, d.At)   # At^ij
    A_mix = np.einsum("kl...,lj...->kj...", ginv, d.At)               # At^k_j
    out = np.empty((NF,) + a.shape)
    out[F_ALPHA] = adv(F_ALPHA, d.d_alpha) - 2.0 * a * K                          # (1)
    f_alpha = prm.lambda_f0 + prm.lambda_f1 * a
    for i in range(3):
        out[F_BETA + i] = adv(F_BETA + i, d.d_beta[:, i]) \
            + 0.75 * f_alpha * d.B[i]                                             # (2)
    rhs_gt = lie(d.gt, d.d_gt, F_GAM) - 2.0 * a * d.At                            # (4)
    out[F_CHI] = adv(F_CHI, d.d_chi) + (2.0 / 3.0) * d.chi * (a * K - div_beta)   # (5)
    rhs_At = (lie(d.At, d.d_At, F_AT) + d.chi * tf(-G["DDa"] + a * G["Ric"])
              + a * (K * d.At - 2.0 * np.einsum("ik...,kj...->ij...", d.At, A_mix)))  # (6)
    out[F_K] = adv(F_K, d.d_K) - G["DDa_tr"] + a * (np.einsum("ij...,ij...->...", d.At, A_up)
                                              + K * K / 3.0)                       # (7)
    # (8) from P:L117-119, reading R7
    dd_beta_div = np.einsum("jkk...->j...", d.dd_beta)                   # d_j d_k beta^k
    rhs_Gt = (np.einsum("jk...,jki...->i...", ginv, d.dd_beta)
              + np.einsum("ij...,j...->i...", ginv, dd_beta_div) / 3.0
              + np.stack([adv(F_GT + i, d.d_Gt[:, i]) for i in range(3)])
              - np.einsum("j...,ji...->i...", CalGt, d.d_beta)
              + (2.0 / 3.0) * CalGt * div_beta
              - 2.0 * np.einsum("ij...,j...->i...", A_up, d.d_alpha)
              + 2.0 * a * (np.einsum("ijk...,jk...->i...", Gam, A_up)
                           - 1.5 / chi * np.einsum("ij...,j...->i...", A_up, d.d_chi)
                           - (2.0 / 3.0) * np.einsum("ij...,j...->i...", ginv, d.d_K)))
    for i in range(3):
        out[F_GT + i] = rhs_Gt[i]
        out[F_B + i] = (rhs_Gt[i] - prm.eta * d.B[i]                               # (3)
                        + adv(F_B + i, d.d_B[:, i])
                        - adv(F_GT + i, d.d_Gt[:, i]))
    out[F_GAM:F_GAM + 6] = full_to_sym(rhs_gt)
    out[F_AT:F_AT + 6] = full_to_sym(rhs_At)
    return out


def rhs_patches(P, h, prm: Params, chunk=512):
    """Full RHS (algebra + KO) at the interior points of patches P [24, n, 13^3].
    Returns [24, n, 7, 7, 7]."""
    P = np.asarray(P).reshape(NF, -1, 13, 13, 13)
    h = np.asarray(h, dtype=np.float64)
    n = P.shape[1]
    out = np.empty((NF, n, 7, 7, 7))
    for i0 in range(0, n, chunk):
        i1 = min(n, i0 + chunk)
        Pc = P[:, i0:i1]
        d = PointData(Pc, h[i0:i1], upwind=bool(prm.upwind))
        r = algebra(d, prm)
        hh = h[i0:i1][:, None, None, None]
        for f in range(NF):
            r[f] += fd.ko_sum(Pc[f], hh, prm.ko_sigma)
        out[:, i0:i1] = r
    return out
