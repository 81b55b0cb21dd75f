"""Symbolic algebraic part A of the BSSN RHS (§III-A eqs (1)-(19),
P:L97-157; §IV-B: "a mapping between 234 (i.e. 24 + 210) inputs to
24 outputs"), for the code generators of gen.py.

Written from the paper with the readings of DESIGN.md §2 (R1 -1/2 on the first
term of eq 17; R2 bracket of eq 19; R3 1/(2 chi) in eq 13; R4 eq 8 from
P:L117-119; R5 Lie weights -2/3 for gt, At and 0 for scalars; R6 f(alpha) =
lambda_f0 + lambda_f1 alpha, eta; R7 CalGt for the undifferentiated Gt; R13 chi
in every division is chi_e = max(chi, chi_floor), an extra kernel-computed
input) and the Kreiss-Oliger terms added after the algebra (R8).  The inverse
conformal metric is the adjugate over the determinant.

Input order (234 + params), the layout of dgr_rhs_inputs / dgr_rhs_algebra:
  [0, 24)     values of the 24 fields (field order of include/dgr.h)
  [24, 96)    d_k f          at 24 + 3 f + k
  [96, 162)   d_k d_l f      at 96 + 6 s + q, s over SECOND = (alpha, chi,
              beta^0..2, gt_xx..gt_zz), q over (xx, xy, xz, yy, yz, zz)
  [162, 234)  KO_k f         at 162 + 3 f + k (already scaled by sigma/(64 h))
"""
from __future__ import annotations

import sympy as sp

NF = 24
SYM = [(0, 0), (0, 1), (0, 2), (1, 1), (1, 2), (2, 2)]
SECOND = [0, 1, 6, 7, 8, 12, 13, 14, 15, 16, 17]
N_IN = 234
NAMES = (["alpha", "chi", "K"] + [f"Gt{i}" for i in range(3)] + [f"beta{i}" for i in range(3)]
         + [f"B{i}" for i in range(3)] + [f"gt{a}{b}" for a, b in SYM]
         + [f"At{a}{b}" for a, b in SYM])


def q_of(i, j):
    return SYM.index((min(i, j), max(i, j)))


def inputs():
    """(symbols [234], params dict).  Symbols are named after their role."""
    v = [sp.Symbol(n, real=True) for n in NAMES]
    d1 = [sp.Symbol(f"d{k}_{NAMES[f]}", real=True) for f in range(NF) for k in range(3)]
    d2 = [sp.Symbol(f"dd{a}{b}_{NAMES[f]}", real=True) for f in SECOND for (a, b) in SYM]
    ko = [sp.Symbol(f"ko{k}_{NAMES[f]}", real=True) for f in range(NF) for k in range(3)]
    syms = v + d1 + d2 + ko
    assert len(syms) == N_IN
    prm = {n: sp.Symbol(n, real=True) for n in ("eta", "lambda_f0", "lambda_f1", "chi_e")}
    return syms, prm


def rhs_exprs(want_geometry=False):
    """The 24 output expressions (field order) and the input symbols (and, with
    want_geometry, the geometric intermediates for other generated kernels)."""
    syms, prm = inputs()
    val = syms[:24]
    D = lambda f, k: syms[24 + 3 * f + k]
    DD = lambda f, a, b: syms[96 + 6 * SECOND.index(f) + q_of(a, b)]
    KO = lambda f: syms[162 + 3 * f] + syms[162 + 3 * f + 1] + syms[162 + 3 * f + 2]
    alpha, chi, K = val[0], val[1], val[2]
    chi_e = prm["chi_e"]                                   # R13
    Gt = val[3:6]
    beta = val[6:9]
    B = val[9:12]
    gt = sp.Matrix(3, 3, lambda i, j: val[12 + q_of(i, j)])
    At = sp.Matrix(3, 3, lambda i, j: val[18 + q_of(i, j)])
    R3 = range(3)
    # inverse conformal metric: adjugate / determinant
    det = gt.det()
    idet = 1 / det
    adj = gt.adjugate()
    gi = sp.Matrix(3, 3, lambda i, j: adj[i, j] * idet)
    dgt = lambda m, i, j: D(12 + q_of(i, j), m)            # d_m gt_ij
    dAt = lambda m, i, j: D(18 + q_of(i, j), m)
    db = lambda j, i: D(6 + i, j)                          # d_j beta^i
    dGt = lambda j, i: D(3 + i, j)                         # d_j Gt^i
    dB = lambda j, i: D(9 + i, j)
    dchi = [D(1, k) for k in R3]
    dalpha = [D(0, k) for k in R3]
    dK = [D(2, k) for k in R3]
    div_beta = sum(db(k, k) for k in R3)
    adv = lambda f: sum(beta[k] * D(f, k) for k in R3)
    # eq (12): first and second kind Christoffel symbols of gt
    C = [[[sp.Rational(1, 2) * (dgt(i, k, j) + dgt(j, k, i) - dgt(k, i, j)) for j in R3]
          for i in R3] for k in R3]
    Gam = [[[sum(gi[k, l] * C[l][i][j] for l in R3) for j in R3] for i in R3] for k in R3]
    CalGt = [sum(gi[i, j] * Gam[k][i][j] for i in R3 for j in R3) for k in R3]   # R7
    # eq (13), reading R3
    gdchi = [sum(gi[k, l] * dchi[l] for l in R3) for k in R3]
    Gphys = [[[Gam[k][i][j] - ((1 if k == i else 0) * dchi[j] + (1 if k == j else 0) * dchi[i]
                               - gt[i, j] * gdchi[k]) / (2 * chi_e)
               for j in R3] for i in R3] for k in R3]
    # eqs (14)-(15)
    DDa = sp.Matrix(3, 3, lambda i, j: DD(0, i, j) - sum(Gphys[k][i][j] * dalpha[k] for k in R3))
    DDa_tr = chi * sum(gi[i, j] * DDa[i, j] for i in R3 for j in R3)
    # eq (17), reading R1; Gt_ijk = gt_il Gt^l_jk
    Gl = [[[sum(gt[i, l] * Gam[l][j][k] for l in R3) for k in R3] for j in R3] for i in R3]

    def Rt(i, j):
        t = -sp.Rational(1, 2) * sum(gi[l, m] * DD(12 + q_of(i, j), l, m) for l in R3 for m in R3)
        t += sp.Rational(1, 2) * sum(gt[k, i] * dGt(j, k) + gt[k, j] * dGt(i, k) for k in R3)
        t += sp.Rational(1, 2) * sum(CalGt[k] * (Gl[i][j][k] + Gl[j][i][k]) for k in R3)
        t += sum(gi[l, m] * (Gam[k][l][i] * Gl[j][k][m] + Gam[k][l][j] * Gl[i][k][m]
                             + Gam[k][i][m] * Gl[k][l][j])
                 for l in R3 for m in R3 for k in R3)
        return t

    # eqs (18)-(19), reading R2
    bracket = (sum(gi[k, l] * DD(1, k, l) for k in R3 for l in R3)
               - sp.Rational(3, 2) / chi_e * sum(gi[k, l] * dchi[k] * dchi[l] for k in R3 for l in R3)
               - sum(CalGt[m] * dchi[m] for m in R3))

    def Rchi(i, j):
        return ((DD(1, i, j) - sum(Gam[k][i][j] * dchi[k] for k in R3)) / (2 * chi_e)
                - dchi[i] * dchi[j] / (4 * chi_e ** 2) + gt[i, j] / (2 * chi_e) * bracket)

    Ric = sp.Matrix(3, 3, lambda i, j: Rt(i, j) + Rchi(i, j) if i <= j else 0)
    for i in R3:
        for j in range(i):
            Ric[i, j] = Ric[j, i]

    def lie(T, dT):                                        # eq (10), R5 weight -2/3
        return sp.Matrix(3, 3, lambda i, j: sum(beta[k] * dT(k, i, j) for k in R3)
                         + sum(T[i, k] * db(j, k) + T[k, j] * db(i, k) for k in R3)
                         - sp.Rational(2, 3) * T[i, j] * div_beta)

    def tf(T):                                             # eq (11)
        tr = sum(gi[l, m] * T[l, m] for l in R3 for m in R3)
        return sp.Matrix(3, 3, lambda i, j: T[i, j] - gt[i, j] * tr / 3)

    A_up = sp.Matrix(3, 3, lambda i, j: sum(gi[i, k] * gi[j, l] * At[k, l] for k in R3 for l in R3))
    A_mix = sp.Matrix(3, 3, lambda k, j: sum(gi[k, l] * At[l, j] for l in R3))
    out = [None] * NF
    out[0] = adv(0) - 2 * alpha * K                                                   # (1)
    f_alpha = prm["lambda_f0"] + prm["lambda_f1"] * alpha
    for i in R3:
        out[6 + i] = sum(beta[j] * db(j, i) for j in R3) + sp.Rational(3, 4) * f_alpha * B[i]   # (2)
    rhs_gt = lie(gt, dgt) - 2 * alpha * At                                            # (4)
    out[1] = adv(1) + sp.Rational(2, 3) * chi * (alpha * K - div_beta)                # (5)
    M6 = tf(-DDa + alpha * Ric)
    rhs_At = sp.Matrix(3, 3, lambda i, j: lie(At, dAt)[i, j] + chi * M6[i, j]
                       + alpha * (K * At[i, j] - 2 * sum(At[i, k] * A_mix[k, j] for k in R3)))  # (6)
    out[2] = adv(2) - DDa_tr + alpha * (sum(At[i, j] * A_up[i, j] for i in R3 for j in R3)
                                        + K * K / 3)                                  # (7)
    dd_beta_div = [sum(DD(6 + k, j, k) for k in R3) for j in R3]
    for i in R3:                                                                      # (8)
        gtr = (sum(gi[j, k] * DD(6 + i, j, k) for j in R3 for k in R3)
               + sum(gi[i, j] * dd_beta_div[j] for j in R3) / 3
               + sum(beta[j] * dGt(j, i) for j in R3)
               - sum(CalGt[j] * db(j, i) for j in R3)
               + sp.Rational(2, 3) * CalGt[i] * div_beta
               - 2 * sum(A_up[i, j] * dalpha[j] for j in R3)
               + 2 * alpha * (sum(Gam[i][j][k] * A_up[j, k] for j in R3 for k in R3)
                              - sp.Rational(3, 2) / chi_e * sum(A_up[i, j] * dchi[j] for j in R3)
                              - sp.Rational(2, 3) * sum(gi[i, j] * dK[j] for j in R3)))
        out[3 + i] = gtr
        out[9 + i] = (gtr - prm["eta"] * B[i] + sum(beta[j] * dB(j, i) for j in R3)   # (3)
                      - sum(beta[j] * dGt(j, i) for j in R3))
    for q, (i, j) in enumerate(SYM):
        out[12 + q] = rhs_gt[i, j]
        out[18 + q] = rhs_At[i, j]
    algebra = list(out)
    with_ko = [algebra[f] + KO(f) for f in range(NF)]
    if want_geometry:
        geo = dict(gi=gi, gt=gt, At=At, K=K, chi_e=chi_e, Gphys=Gphys, Ric=Ric, D=D,
                   dgt=dgt, dAt=dAt, dchi=dchi, dK=dK)
        return with_ko, syms, prm, geo
    return with_ko, syms, prm
