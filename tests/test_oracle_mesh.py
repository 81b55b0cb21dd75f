"""Pins for oracle/octree.py and oracle/maps.py.

Closed forms and brute force on tiny trees (SURVEY.md §8c pins, "Octree"):
* uniform trees: (6*2^l + 1)^3 DOFs (non-periodic) / (6*2^l)^3 (periodic), no hanging;
* refinement rule: every leaf is at or above its target, every split parent was below it;
* 2:1 vertex balance, completeness, Morton order, local minimality of the closure;
* DOF classification, first-sight numbering, hanging sources, zip owners and
  padding sources recomputed by pure-Python brute force over all leaves.
"""
import itertools

import numpy as np
import pytest

from oracle import octree
from oracle.maps import (K, KIND_COPY, KIND_EXTRAP, KIND_INJECT, KIND_INTERP, KIND_SELF,
                         KIND_WRAP, OracleMesh)
from synth import configs
from synth.configs import MeshConfig, Puncture


def tiny(periodic=False, lmax=3, rho=0.15, lmin=1, seed=0, two=False):
    rng = np.random.default_rng(seed)
    pts = [Puncture(*rng.uniform(-0.3, 0.3, size=3), 1.0, lmax)]
    if two:
        pts.append(Puncture(*rng.uniform(-0.4, 0.4, size=3), 0.5, lmax - 1))
    return MeshConfig(name="tiny", xmin=(-1.0, -1.0, -1.0), width=2.0, periodic=periodic,
                      level_min=lmin, punctures=tuple(pts), rho=rho)


def test_uniform_counts():
    m = OracleMesh(configs.c1_uniform())
    m.build_dofs()
    assert m.n_oct == 512 and m.n_dof == 48 ** 3
    assert m.is_dof.all()
    cfg = MeshConfig(name="u2", xmin=(0, 0, 0), width=1.0, periodic=False, level_min=2)
    m2 = OracleMesh(cfg)
    m2.build_dofs()
    assert m2.n_oct == 64 and m2.n_dof == 25 ** 3 and m2.is_dof.all()


@pytest.mark.parametrize("name", ["small", "small_bbh", "c2"])
def test_refinement_rule(name):
    cfg = configs.get(name)
    a, l = octree.refine(cfg)
    tgt = octree.target_levels(a, l, cfg)
    assert np.all(l >= tgt)
    # the parent of every leaf was split because it was below its own target
    D = cfg.max_depth
    ps = (np.int64(1) << (D - l + 1))
    pa = (a // ps[:, None]) * ps[:, None]
    nz = l > 0
    ptgt = octree.target_levels(pa[nz], l[nz] - 1, cfg)
    assert np.all(l[nz] - 1 < ptgt)


@pytest.mark.parametrize("periodic", [False, True])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_balance_bruteforce(periodic, seed):
    cfg = tiny(periodic=periodic, seed=seed, two=True, lmax=4, rho=0.08)
    a, l = octree.build_octree(cfg)
    D = cfg.max_depth
    assert octree.is_complete(a, l, D)
    keys = octree.morton_key(a[:, 0], a[:, 1], a[:, 2], D)
    assert np.all(np.diff(keys) > 0)
    assert octree.is_balanced_bruteforce(a, l, D, periodic)
    # local minimality: merging any 8 sibling leaves that balancing created
    # (their parent was not split by the refinement rule) breaks the balance
    ra, rl = octree.refine(cfg)
    ref = set(zip(map(tuple, ra.tolist()), rl.tolist()))
    internal_ref = set()
    for (an, lv) in ref:
        for L in range(lv):
            s = 1 << (D - L)
            internal_ref.add((tuple((np.array(an) // s) * s), L))
    groups = {}
    for i in range(len(l)):
        if l[i] == 0:
            continue
        s = 1 << (D - int(l[i]) + 1)
        par = (tuple((a[i] // s) * s), int(l[i]) - 1)
        groups.setdefault(par, []).append(i)
    n_checked = 0
    for par, kids in groups.items():
        if len(kids) != 8 or par in internal_ref:
            continue
        keep = np.ones(len(l), dtype=bool)
        keep[kids] = False
        na = np.concatenate([a[keep], np.array([par[0]])])
        nl = np.concatenate([l[keep], np.array([par[1]])])
        assert not octree.is_balanced_bruteforce(na, nl, D, periodic), par
        n_checked += 1
    assert n_checked >= 0


def test_balance_adds_octants_when_needed():
    """A hand-made violation: one level-3 leaf inside a level-1 tree."""
    D = 18
    cfg = MeshConfig(name="h", xmin=(0, 0, 0), width=1.0, periodic=False, level_min=1)
    a, l = octree.refine(cfg)
    # refine child 0 twice at its corner -> a level-3 leaf next to level-1 leaves
    a1, l1 = octree.children(a[:1], l[:1], D)
    a2, l2 = octree.children(a1[7:8], l1[7:8], D)
    A = np.concatenate([a[1:], a1[:7], a2])
    Lv = np.concatenate([l[1:], l1[:7], l2])
    assert not octree.is_balanced_bruteforce(A, Lv, D, False)
    B, Lb = octree.balance(A, Lv, D, False)
    assert octree.is_balanced_bruteforce(B, Lb, D, False)
    assert octree.is_complete(B, Lb, D)
    assert len(Lb) > len(Lv)


# ----------------------------------------------------------- brute force maps

def _boxes(m):
    lo = 6 * m.anchors
    hi = lo + 6 * m.side[:, None]
    return lo, hi


def _contains(m, X):
    """All (leaf, shift) whose closed box contains lattice point X."""
    lo, hi = _boxes(m)
    L = m.L
    shifts = np.array(list(itertools.product(*([(-L, 0, L)] * 3))) if m.periodic
                      else [(0, 0, 0)], dtype=np.int64)
    # [shift, leaf]: every leaf tested against every periodic image (vectorised brute force)
    inside = np.all((lo[None] + shifts[:, None] <= X) & (X <= hi[None] + shifts[:, None]), axis=2)
    out = []
    for c in range(m.n_oct):
        hit = np.nonzero(inside[:, c])[0]
        if len(hit):
            out.append((c, shifts[hit[0]]))
    return out


def _on_grid(m, X, c, s):
    return np.all((X - s - 6 * m.anchors[c]) % m.side[c] == 0)


@pytest.mark.parametrize("periodic", [False, True])
def test_dofs_bruteforce(periodic):
    cfg = tiny(periodic=periodic, lmax=3, rho=0.05, seed=3)
    m = OracleMesh(cfg)
    assert 15 <= m.n_oct <= 120
    m.build_dofs()
    ids = {}
    o2n = np.full((m.n_oct, 343), -1)
    n_hang = 0
    for e in range(m.n_oct):
        for n in range(343):
            ijk = np.array([n % 7, (n // 7) % 7, n // 49])
            X = 6 * m.anchors[e] + ijk * m.side[e]
            Xw = X % m.L if periodic else X
            cont = _contains(m, Xw)
            if all(_on_grid(m, Xw, c, s) for c, s in cont):
                key = tuple(Xw)
                if key not in ids:
                    ids[key] = len(ids)
                o2n[e, n] = ids[key]
                # zip owner (R17): coarsest, then lowest index
                own = min(cont, key=lambda cs: (m.levels[cs[0]], cs[0]))[0]
                assert m.zip_leaf[ids[key]] == own
            else:
                n_hang += 1
                src = min(c for c, s in cont if m.levels[c] < m.levels[e])
                assert m.hang_src[e, n] == src
    assert np.array_equal(o2n, m.o2n)
    assert m.n_dof == len(ids)
    assert n_hang == int((~m.is_dof).sum()) and n_hang > 0


@pytest.mark.parametrize("periodic", [False, True])
def test_padding_sources_bruteforce(periodic):
    cfg = tiny(periodic=periodic, lmax=3, rho=0.05, seed=4)
    m = OracleMesh(cfg)
    lo, hi = _boxes(m)
    # octants with the most varied neighbourhoods: each level, near the boundary and not
    rng = np.random.default_rng(0)
    octs = sorted(set(rng.choice(m.n_oct, size=6, replace=False).tolist()
                      + [int(np.argmax(m.levels)), int(np.argmin(m.levels))]))
    src, kind = m.padding_sources(octs)
    seen = set()
    for row, b in enumerate(octs):
        for p in range(13 ** 3):
            ijk = np.array([p % 13, (p // 13) % 13, p // 169])
            X = 6 * m.anchors[b] + (ijk - K) * m.side[b]
            if np.all((ijk >= K) & (ijk < K + 7)):
                assert src[row, p] == b and kind[row, p] == KIND_SELF
                continue
            if not periodic and np.any((X < 0) | (X > m.L)):
                assert src[row, p] == -1 and kind[row, p] == KIND_EXTRAP
                seen.add(KIND_EXTRAP)
                continue
            best = None
            for c, s in _contains(m, X % m.L if periodic else X):
                sh = s + (X - (X % m.L) if periodic else 0)
                if np.all(lo[c] + sh <= hi[b]) and np.all(lo[b] <= hi[c] + sh):
                    k = (-m.levels[c], c)
                    if best is None or k < best[0]:
                        best = (k, c, np.any(sh != 0))
            assert best is not None
            _, c, wrapped = best
            lv = m.levels
            kd = KIND_COPY if lv[c] == lv[b] else (KIND_INJECT if lv[c] > lv[b] else KIND_INTERP)
            if wrapped:
                kd |= KIND_WRAP
            assert src[row, p] == c, (b, p)
            assert kind[row, p] == kd, (b, p, kind[row, p], kd)
            seen.add(kd & 7)
    assert {KIND_COPY} <= seen
