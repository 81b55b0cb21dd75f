"""Pins of the oracle's Sommerfeld radiative outer boundary (reading R29,
oracle/boundary.py) against what the mathematics fixes:
the condition is exact for outgoing spherical waves and violated by incoming
ones; flat data has zero RHS; it acts on exactly the DOFs on the domain faces
(closed-form count) and nowhere else; and on data of degree <= 6 per axis the
oracle's finite-difference version (centred D1 on the extrapolated padding)
equals the condition with exact derivatives."""
import numpy as np
import pytest

from oracle import boundary as obc
from oracle import bssn, rk4
from oracle.maps import OracleMesh
from synth import initial
from synth.configs import MeshConfig


def _wave(x, t, sign):
    """f = f_inf + g(r - sign t)/r with g(s) = exp(-(s - 3)^2); exact d_t f, grad f."""
    r = np.sqrt((x * x).sum(axis=0))
    s = r - sign * t
    g = np.exp(-(s - 3.0) ** 2)
    dg = -2.0 * (s - 3.0) * g
    f = 0.7 + g / r
    dfdr = dg / r - g / (r * r)
    grad = x / r * dfdr
    dt = -sign * dg / r
    return f, grad, dt


def test_outgoing_spherical_wave_is_exact():
    rng = np.random.default_rng(0)
    x = rng.uniform(-6.0, 6.0, size=(3, 200))
    x[:, np.sqrt((x * x).sum(axis=0)) < 0.5] += 1.0
    f, grad, dt = _wave(x, 0.4, +1)
    got = obc.sommerfeld_rhs(f, grad, x, 0.7)
    assert np.max(np.abs(got - dt)) <= 1e-14 * np.max(np.abs(dt)) + 1e-15


def test_incoming_spherical_wave_violates_it():
    rng = np.random.default_rng(1)
    x = rng.uniform(2.0, 6.0, size=(3, 200))
    f, grad, dt = _wave(x, 0.4, -1)
    got = obc.sommerfeld_rhs(f, grad, x, 0.7)
    assert np.max(np.abs(got - dt)) > 0.1 * np.max(np.abs(dt))


def _uniform(level=2, w=2.0):
    cfg = MeshConfig(name="uniform_np", xmin=(-w / 2,) * 3, width=w, periodic=False,
                     level_min=level, punctures=(), description="uniform non-periodic")
    om = OracleMesh(cfg)
    om.build_dofs()
    return cfg, om


def test_flat_data_zero_rhs_with_sommerfeld():
    cfg, om = _uniform()
    u = initial.minkowski(om.dof_coords())
    r = rk4.rhs_dofs(om, u, bssn.Params(sommerfeld=1))
    assert np.all(r == 0.0)


def test_acts_on_exactly_the_face_dofs():
    cfg, om = _uniform(level=2)
    x = om.dof_coords()
    u = initial.for_config(cfg, x, kind="random", seed=4)
    r0 = rk4.rhs_dofs(om, u, bssn.Params())
    r1 = rk4.rhs_dofs(om, u, bssn.Params(sommerfeld=1))
    lo = np.asarray(cfg.xmin)[:, None]
    hi = lo + cfg.width
    face = np.any((x == lo) | (x == hi), axis=0)
    n = 6 * 4 + 1                                    # nodes per edge at level 2
    assert face.sum() == n ** 3 - (n - 2) ** 3
    assert np.array_equal(r0[:, ~face], r1[:, ~face])
    assert np.all(np.any(r0[:, face] != r1[:, face], axis=0))


def test_fd_version_exact_on_degree_six_data():
    """alpha = 1 + a x^3 + b y^2 z^4 (degree <= 6 per axis), other fields flat:
    the centred D1 on the extrapolated padding is exact, so at every face DOF
    the oracle's RHS of alpha equals the condition with the exact gradient."""
    cfg, om = _uniform(level=2)
    x = om.dof_coords()
    u = initial.minkowski(x)
    a, b = 0.03, -0.02
    X, Y, Z = x
    u[bssn.F_ALPHA] = 1.0 + a * X ** 3 + b * Y ** 2 * Z ** 4
    grad = np.stack([3 * a * X ** 2, 2 * b * Y * Z ** 4, 4 * b * Y ** 2 * Z ** 3])
    r = rk4.rhs_dofs(om, u, bssn.Params(sommerfeld=1))
    lo = np.asarray(cfg.xmin)[:, None]
    face = np.any((x == lo) | (x == lo + cfg.width), axis=0)
    exact = obc.sommerfeld_rhs(u[bssn.F_ALPHA][face], grad[:, face], x[:, face], 1.0)
    err = np.max(np.abs(r[bssn.F_ALPHA][face] - exact))
    assert err <= 1e-11 * np.max(np.abs(exact)), err


def test_periodic_domain_is_untouched():
    from synth import configs
    cfg = configs.c1_uniform()
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords(), kind="random", seed=2)
    octs = np.arange(4)
    P = np.zeros((24, 4, 13, 13, 13))
    r = np.ones((24, 4, 7, 7, 7))
    assert obc.apply_sommerfeld(om, octs, P, r) is r
