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

import multiprocessing as mp
import os

import numpy as np

from .boundary import apply_sommerfeld
from .bssn import NF, Params, rhs_patches
from .maps import OracleMesh
from .unzip import elements, padding_sources_cached, unzip, unzip_from_elements, zip_rhs

COURANT = 0.25


def octant_h(mesh: OracleMesh):
    return mesh.cfg.width / (6.0 * (2.0 ** mesh.levels))


def rhs_dofs(mesh: OracleMesh, u: np.ndarray, prm: Params, workers=None) -> np.ndarray:
    """F(u): [24, n_dof] -> [24, n_dof].

    workers > 1 evaluates octant-to-patch + RHS on chunks of octants in forked
    worker processes (the element reconstruction, which couples octants, is
    done once in the parent); the arithmetic per octant is unchanged.
    Default: $DGR_ORACLE_WORKERS, else 1."""
    if workers is None:
        workers = int(os.environ.get("DGR_ORACLE_WORKERS", "1"))
    if workers <= 1 or mesh.n_oct < 4 * workers:
        P = unzip(mesh, u)
        r = rhs_patches(P, octant_h(mesh), prm)
        if prm.sommerfeld:
            r = apply_sommerfeld(mesh, np.arange(mesh.n_oct), P, r)
        return zip_rhs(mesh, r.reshape(NF, mesh.n_oct, 343))
    E = elements(mesh, u)
    padding_sources_cached(mesh, np.arange(1))          # fill the cache before forking
    _G.update(mesh=mesh, E=E, prm=prm)
    nch = 4 * workers
    bounds = np.linspace(0, mesh.n_oct, nch + 1).astype(int)
    chunks = [(int(a), int(b)) for a, b in zip(bounds[:-1], bounds[1:]) if b > a]
    with mp.get_context("fork").Pool(workers) as pool:
        parts = pool.map(_chunk_rhs, chunks)
    _G.clear()
    r = np.empty((NF, mesh.n_oct, 343))
    for a, rr in parts:
        r[:, a:a + rr.shape[1]] = rr
    return zip_rhs(mesh, r)


_G = {}


def _chunk_rhs(ab):
    from threadpoolctl import threadpool_limits
    a, b = ab
    mesh, E, prm = _G["mesh"], _G["E"], _G["prm"]
    octs = np.arange(a, b)
    with threadpool_limits(limits=1):
        P = unzip_from_elements(mesh, E, octs)
        r = rhs_patches(P, octant_h(mesh)[octs], prm)
        if prm.sommerfeld:
            r = apply_sommerfeld(mesh, octs, P, r)
    return a, r.reshape(NF, len(octs), 343)


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
