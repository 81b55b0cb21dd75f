"""Symbolic Weyl scalar Psi_4 from the BSSN variables and their derivatives
(readings R33-R34 of DESIGN.md, the standard 3+1 forms of the
paper's reference [44]), for the generated kernel k_psi4 (gen.py):

  gamma_ij = gt_ij / chi_e, K_ij = (At_ij + gt_ij K / 3) / chi_e,
  E_ij = R_ij + K K_ij - K_ik gamma^kl K_lj,
  B_ij = (eps_i^kl D_k K_lj + eps_j^kl D_k K_li) / 2,  eps^mkl = [mkl] / sqrt(gamma),
  tetrad: r^, theta^, phi^ about the extraction centre, Gram-Schmidt in gamma,
  Psi_4 = (E_ij - i B_ij) mbar^i mbar^j, mbar = (e_theta - i e_phi) / sqrt(2).

Inputs: the 234 of bssn_sym (values and derivatives) + the point's position
(x, y, z) relative to the extraction centre; outputs (Re Psi_4, Im Psi_4).
The Ricci tensor and Christoffels are bssn_sym's (eqs 13, 16-19)."""
from __future__ import annotations

import sympy as sp

from . import bssn_sym

LEVI = {(0, 1, 2): 1, (1, 2, 0): 1, (2, 0, 1): 1, (0, 2, 1): -1, (2, 1, 0): -1, (1, 0, 2): -1}


def psi4_exprs():
    _, syms, prm, g = bssn_sym.rhs_exprs(want_geometry=True)
    x, y, z = sp.symbols("px py pz", real=True)
    R3 = range(3)
    chi_e, gt, At, K, gi = g["chi_e"], g["gt"], g["At"], g["K"], g["gi"]
    gam = gt / chi_e
    gam_inv = gi * chi_e
    Kij = (At + gt * K / 3) / chi_e
    dchi, dK = g["dchi"], g["dK"]

    def dKij(k, i, j):   # d_k K_ij, product rule
        return ((g["dAt"](k, i, j) + g["dgt"](k, i, j) * K / 3 + gt[i, j] * dK[k] / 3) / chi_e
                - (At[i, j] + gt[i, j] * K / 3) * dchi[k] / chi_e ** 2)

    Gp = g["Gphys"]                                         # Gp[m][k][l] = Gamma^m_kl
    DK = [[[dKij(k, l, j) - sum(Gp[m][k][l] * Kij[m, j] for m in R3)
            - sum(Gp[m][k][j] * Kij[l, m] for m in R3) for j in R3] for l in R3] for k in R3]
    trK = sum(gam_inv[i, j] * Kij[i, j] for i in R3 for j in R3)
    E = sp.Matrix(3, 3, lambda i, j: g["Ric"][i, j] + trK * Kij[i, j]
                  - sum(Kij[i, k] * gam_inv[k, l] * Kij[l, j] for k in R3 for l in R3))
    sqg = sp.sqrt(gt.det() / chi_e ** 3)
    eps_mix = lambda i, k, l: sum(gam[i, m] * LEVI.get((m, k, l), 0) for m in R3) / sqg
    Bh = sp.Matrix(3, 3, lambda i, j: sum(eps_mix(i, k, l) * DK[k][l][j] for k in R3 for l in R3))
    B = (Bh + Bh.T) / 2
    r = sp.sqrt(x * x + y * y + z * z)
    rho = sp.sqrt(x * x + y * y)
    v = [sp.Matrix([x, y, z]) / r, sp.Matrix([x * z, y * z, -(x * x + y * y)]) / (r * rho),
         sp.Matrix([-y, x, 0]) / rho]
    dot = lambda a, b: (a.T * gam * b)[0, 0]
    e = []
    for w in v:
        for u in e:
            w = w - dot(u, w) * u
        e.append(w / sp.sqrt(dot(w, w)))
    et, ep = e[1], e[2]
    P = sp.Matrix(3, 3, lambda i, j: (et[i] * et[j] - ep[i] * ep[j]) / 2)       # Re mbar mbar
    Q = sp.Matrix(3, 3, lambda i, j: -(et[i] * ep[j] + ep[i] * et[j]) / 2)      # Im mbar mbar
    re = sum(E[i, j] * P[i, j] + B[i, j] * Q[i, j] for i in R3 for j in R3)
    im = sum(E[i, j] * Q[i, j] - B[i, j] * P[i, j] for i in R3 for j in R3)
    return [re, im], syms, prm, (x, y, z)
