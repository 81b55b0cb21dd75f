"""Workload descriptors (mesh-generation inputs) shared by tests, bench and both
sides of every parity check.

This module holds NO arithmetic of the method: it only states the inputs —
domain, boundary mode, coarsest level, punctures (position, mass, finest level)
and the refinement radius factor rho — for the five BASELINE.json configs.

Refinement rule (a [proposed] reading; the paper's WAMR
tolerance ε, cannot be reproduced without Dendro-GR): every
octant o is refined while level(o) < target(o), with
    target(o) = max(l_min, max_a [L_a - j_a(o)]),
    j_a(o) = smallest j >= 0 with d^2(o, x_a) <= (rho*m_a)^2 * 4^j,
d = distance from x_a to o's closed box.  Both implementations (oracle/ and
libdgr) evaluate it themselves from these numbers.

Mass/position conventions: total mass 1, m1 = q/(1+q),
m2 = 1/(1+q), separation 8 along x (Table I caption), centre of
mass at the origin, finest level at the smaller hole m2 (reading R20),
punctures offset by +h_min/4 in z so no grid node coincides with a puncture.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List, Tuple

MAX_DEPTH = 18          # anchors are integers in [0, 2^18) per axis


@dataclass(frozen=True)
class Puncture:
    x: float
    y: float
    z: float
    m: float
    level: int          # finest level required at the puncture


@dataclass(frozen=True)
class MeshConfig:
    name: str
    xmin: Tuple[float, float, float]
    width: float
    periodic: bool
    level_min: int
    punctures: Tuple[Puncture, ...] = ()
    rho: float = 1.0
    max_depth: int = MAX_DEPTH
    description: str = ""

    @property
    def level_max_nominal(self) -> int:
        return max([self.level_min] + [p.level for p in self.punctures])

    @property
    def h_min(self) -> float:
        return self.width / (6.0 * (1 << self.level_max_nominal))


def _bbh(name: str, q: float, l1: int, l2: int, rho: float, desc: str,
         level_min: int = 3, width: float = 800.0) -> MeshConfig:
    m1 = q / (1.0 + q)
    m2 = 1.0 / (1.0 + q)
    x1 = 8.0 / (1.0 + q)
    x2 = -8.0 * q / (1.0 + q)
    lmax = max(l1, l2, level_min)
    dz = width / (6.0 * (1 << lmax)) / 4.0
    return MeshConfig(
        name=name, xmin=(-width / 2, -width / 2, -width / 2), width=width,
        periodic=False, level_min=level_min,
        punctures=(Puncture(x1, 0.0, dz, m1, l1), Puncture(x2, 0.0, dz, m2, l2)),
        rho=rho, description=desc)


def c1_uniform() -> MeshConfig:
    """configs[0]: uniform level-3 periodic cube [-0.5,0.5]^3, 512 octants, h=1/48."""
    return MeshConfig(name="c1", xmin=(-0.5, -0.5, -0.5), width=1.0, periodic=True,
                      level_min=3, description="uniform level 3, periodic, 512 octants")


def c2_schwarzschild(rho: float = 1.0, lmax: int = 8) -> MeshConfig:
    """configs[1]: single puncture m=1, [-32,32]^3, levels 3..8 (6 AMR levels)."""
    w = 64.0
    dz = w / (6.0 * (1 << lmax)) / 4.0
    return MeshConfig(name="c2", xmin=(-32.0, -32.0, -32.0), width=w, periodic=False,
                      level_min=3, punctures=(Puncture(0.0, 0.0, dz, 1.0, lmax),),
                      rho=rho, description="Schwarzschild puncture m=1, levels 3..%d" % lmax)


def c3_bbh_q1(rho: float = 2.5) -> MeshConfig:
    """configs[2]: BL q=1, levels 3..12 ('9 levels, coarsest 3, finest 12')."""
    return _bbh("c3", 1.0, 12, 12, rho, "BL q=1, levels 3..12, rho=%g" % rho)


def c4_bbh_q4(rho: float = 1.0) -> MeshConfig:
    """configs[3]: BL q=4, finest 15 at m2, 12 at m1 (Fig. 1 shape)."""
    return _bbh("c4", 4.0, 12, 15, rho, "BL q=4, levels 3..15, rho=%g" % rho)


def c5_bbh_q8(rho: float = 1.0) -> MeshConfig:
    """configs[4]: BL q=8, finest 16 at m2, 12 at m1 (Table IV dx 2.03e-3)."""
    return _bbh("c5", 8.0, 12, 16, rho, "BL q=8, levels 3..16, rho=%g" % rho)


def small_adaptive(lmax: int = 6, rho: float = 0.5) -> MeshConfig:
    """A small adaptive puncture mesh (a few hundred octants) for oracle-speed tests."""
    w = 16.0
    dz = w / (6.0 * (1 << lmax)) / 4.0
    return MeshConfig(name="small", xmin=(-8.0, -8.0, -8.0), width=w, periodic=False,
                      level_min=2, punctures=(Puncture(0.3, -0.2, dz, 1.0, lmax),),
                      rho=rho, description="small adaptive puncture mesh")


def small_bbh(lmax: int = 6, rho: float = 0.5) -> MeshConfig:
    """Two punctures of unequal finest level on a small domain (chains of hanging nodes)."""
    return _bbh("small_bbh", 2.0, lmax - 1, lmax, rho, "small q=2 BBH", level_min=2, width=32.0)


def c3_large() -> MeshConfig:
    """configs[2] at the Fig. 17 caption size: BL q=1, levels 3..12, rho = 3.4
    (~257M unknowns; reading R22)."""
    c = c3_bbh_q1(rho=3.4)
    return MeshConfig(**{**c.__dict__, "name": "c3big"})


def table3_mesh(k: int) -> MeshConfig:
    """m1..m5 of PAPER.md Table III: BL q=1 puncture meshes of
    decreasing adaptivity, finest level 12, 10, 8, 6, 4 (levels 3..L, rho 2.5)."""
    L = [12, 10, 8, 6, 4][k - 1]
    c = _bbh("m%d" % k, 1.0, L, L, 2.5, "Table III m%d: BL q=1, levels 3..%d" % (k, L))
    return c


CONFIGS = {
    "c1": c1_uniform,
    "c2": c2_schwarzschild,
    "c3": c3_bbh_q1,
    "c4": c4_bbh_q4,
    "c5": c5_bbh_q8,
    "small": small_adaptive,
    "small_bbh": small_bbh,
    "c3big": c3_large,
    "m1": lambda: table3_mesh(1), "m2": lambda: table3_mesh(2), "m3": lambda: table3_mesh(3),
    "m4": lambda: table3_mesh(4), "m5": lambda: table3_mesh(5),
}


def get(name: str, **kw) -> MeshConfig:
    return CONFIGS[name](**kw)
