"""Seeded synthetic inputs: initial data evaluated at DOF coordinates.

Input generators only — no arithmetic of the method (no derivatives, no RHS).
Used identically by tests, bench and both sides of every parity check.
Field order: 0 alpha, 1 chi, 2 K, 3-5 Gt^i, 6-8 beta^i, 9-11 B^i,
12-17 gt_ij, 18-23 At_ij with ij in (xx, xy, xz, yy, yz, zz).

Recipes:
  minkowski     alpha = chi = 1, gt = delta, rest 0
  brill_lindquist  psi = 1 + sum m_a / (2|x - x_a|); chi = psi^-4; alpha = psi^-2;
                gt = delta; K = At = Gt = beta = B = 0
  gauge_wave    Apples-with-Apples gauge wave at t = 0 (H = 1 - A sin(2 pi x / d))
  random_smooth each field f0 + amp * sum_modes a sin(2 pi k.x / W + phi), |k_i| <= 2
  noise         uniform robust-stability noise of a given amplitude
"""
from __future__ import annotations

import numpy as np

NF = 24
SYM = [(0, 0), (0, 1), (0, 2), (1, 1), (1, 2), (2, 2)]


def minkowski(xyz):
    n = xyz.shape[1]
    u = np.zeros((NF, n))
    u[0] = 1.0
    u[1] = 1.0
    for q, (i, j) in enumerate(SYM):
        if i == j:
            u[12 + q] = 1.0
    return u


def brill_lindquist(xyz, punctures):
    """punctures: iterable of objects with x, y, z, m."""
    psi = np.ones(xyz.shape[1])
    for p in punctures:
        r = np.sqrt((xyz[0] - p.x) ** 2 + (xyz[1] - p.y) ** 2 + (xyz[2] - p.z) ** 2)
        psi = psi + p.m / (2.0 * r)
    u = minkowski(xyz)
    u[1] = psi ** -4
    u[0] = psi ** -2
    return u


def gauge_wave(xyz, amp=0.1, d=1.0):
    ph = 2.0 * np.pi * xyz[0] / d
    H = 1.0 - amp * np.sin(ph)
    dHdx = -amp * np.cos(ph) * 2.0 * np.pi / d
    u = np.zeros((NF, xyz.shape[1]))
    chi = H ** (-1.0 / 3.0)
    Kxx = -(np.pi * amp / d) * np.cos(ph) / np.sqrt(H)
    K = Kxx / H
    u[0] = np.sqrt(H)
    u[1] = chi
    u[2] = K
    u[3] = (2.0 / 3.0) * H ** (-5.0 / 3.0) * dHdx
    u[12 + 0] = H ** (2.0 / 3.0)
    u[12 + 3] = H ** (-1.0 / 3.0)
    u[12 + 5] = H ** (-1.0 / 3.0)
    # At_ij = chi (K_ij - gamma_ij K / 3), gamma = diag(H, 1, 1)
    u[18 + 0] = chi * (Kxx - H * K / 3.0)
    u[18 + 3] = chi * (0.0 - K / 3.0)
    u[18 + 5] = chi * (0.0 - K / 3.0)
    return u


def random_smooth(xyz, width, seed, amp=0.1, nmodes=3, xmin=(0.0, 0.0, 0.0)):
    rng = np.random.default_rng(seed)
    base = minkowski(xyz)
    u = np.empty_like(base)
    x = [(xyz[a] - xmin[a]) / width for a in range(3)]
    for f in range(NF):
        v = base[f].copy()
        for _ in range(nmodes):
            k = rng.integers(-2, 3, size=3)
            a = rng.uniform(-1.0, 1.0)
            phi = rng.uniform(0.0, 2.0 * np.pi)
            v += amp * a * np.sin(2.0 * np.pi * (k[0] * x[0] + k[1] * x[1] + k[2] * x[2]) + phi)
        u[f] = v
    return u


def noise(n, amp, seed):
    rng = np.random.default_rng(seed)
    return rng.uniform(-amp, amp, size=(NF, n))


def for_config(cfg, xyz, kind=None, seed=0):
    """Default initial data of a MeshConfig: BL when it has punctures,
    random smooth otherwise (or `kind` = minkowski|gauge_wave|random|bl)."""
    if kind is None:
        kind = "bl" if cfg.punctures else "random"
    if kind == "bl":
        return brill_lindquist(xyz, cfg.punctures)
    if kind == "minkowski":
        return minkowski(xyz)
    if kind == "gauge_wave":
        return gauge_wave(xyz, amp=0.1, d=cfg.width)
    if kind == "random":
        return random_smooth(xyz, cfg.width, seed, xmin=cfg.xmin)
    raise ValueError(kind)
