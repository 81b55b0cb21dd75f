"""ORACLE (test infrastructure only): one RHS evaluation on DOFs and the
classic RK4 step.

PAPER.md Alg. 1 (L200-227): octant-to-patch -> RHS -> patch-to-octant ->
AXPY; L95: "RK4 with a Courant factor of lambda = 0.25 ... global
timestepping".  Reading R11: the classic tableau
    k1 = F(u), k2 = F(u + dt/2 k1), k3 = F(u + dt/2 k2), k4 = F(u + dt k3),
    u^{n+1} = u + dt/6 (k1 + 2 k2 + 2 k3 + k4),
with dt = 0.25 * h_min.  Only DOFs are evolved; hanging values are rebuilt
by every unzip.
"""
from __future__ import annotations

import numpy as np

from .bssn import NF, Params, rhs_patches
from .maps import OracleMesh
from .unzip import unzip, zip_rhs

COURANT = 0.25


def octant_h(mesh: OracleMesh):
    return mesh.cfg.width / (6.0 * (2.0 ** mesh.levels))


def rhs_dofs(mesh: OracleMesh, u: np.ndarray, prm: Params) -> np.ndarray:
    """F(u): [24, n_dof] -> [24, n_dof]."""
    P = unzip(mesh, u)
    r = rhs_patches(P, octant_h(mesh), prm)
    return zip_rhs(mesh, r.reshape(NF, mesh.n_oct, 343))


def rk4_step(mesh: OracleMesh, u: np.ndarray, dt: float, prm: Params) -> np.ndarray:
    return rk4_step_generic(lambda v: rhs_dofs(mesh, v, prm), u, dt)


def rk4_step_generic(F, u, dt):
    """Classic RK4 for an autonomous F (pinned on u' = lambda u in tests)."""
    k1 = F(u)
    k2 = F(u + 0.5 * dt * k1)
    k3 = F(u + 0.5 * dt * k2)
    k4 = F(u + dt * k3)
    return u + (dt / 6.0) * (k1 + 2.0 * k2 + 2.0 * k3 + k4)


def dt_courant(mesh: OracleMesh) -> float:
    return COURANT * float(octant_h(mesh).min())
