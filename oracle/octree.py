"""ORACLE (test infrastructure only): linear octree construction.

Follows:
  * PAPER.md L168 (§III-B): only leaves are stored; a 2:1 balance constraint is
    enforced ("all its neighbors can differ by at most a single level", L241);
    leaves are ordered along a space-filling curve.
  * SURVEY.md §8c-O1 [proposed]: the distance-graded refinement rule and the
    minimal 2:1 *vertex* balance closure; Morton order with child index
    c = x + 2y + 4z (x least significant in each bit triple).

Anchors are integer coordinates in units of width/2^D (D = max_depth); a level-l
octant has side s = 2^(D-l) in those units.

Everything here is deliberately naive: the refinement is evaluated octant by
octant level by level, and the balance closure is "split every leaf that is two
or more levels coarser than a leaf it touches, repeat until nothing changes",
which is the definition of the minimal closure.
"""
from __future__ import annotations

import numpy as np

# ---------------------------------------------------------------- Morton keys

def morton_key(x, y, z, depth: int):
    """Interleave bits: bit b of x -> key bit 3b, y -> 3b+1, z -> 3b+2."""
    x = np.asarray(x, dtype=np.int64)
    y = np.asarray(y, dtype=np.int64)
    z = np.asarray(z, dtype=np.int64)
    key = np.zeros(np.broadcast(x, y, z).shape, dtype=np.int64)
    for b in range(depth):
        key |= ((x >> b) & 1) << (3 * b)
        key |= ((y >> b) & 1) << (3 * b + 1)
        key |= ((z >> b) & 1) << (3 * b + 2)
    return key


def sort_morton(anchors: np.ndarray, levels: np.ndarray, depth: int):
    keys = morton_key(anchors[:, 0], anchors[:, 1], anchors[:, 2], depth)
    order = np.argsort(keys, kind="stable")
    return anchors[order], levels[order]


# ---------------------------------------------------------- refinement target

def target_levels(anchors: np.ndarray, levels: np.ndarray, cfg) -> np.ndarray:
    """target(o) = max(l_min, max_a [L_a - j_a(o)]), SURVEY.md §8c-O1.

    Exact evaluation order (shared by contract with the C++ builder, which
    implements it independently): unit = width * 2^-D;
    lo = xmin + anchor*unit, hi = xmin + (anchor+side)*unit;
    dx = max(lo - p, 0, p - hi); d2 = (dx*dx + dy*dy) + dz*dz;
    r2 = (rho*m)*(rho*m); j = smallest j>=0 with d2 <= r2 * 4^j.
    """
    D = cfg.max_depth
    unit = cfg.width * 2.0 ** (-D)
    side = (np.int64(1) << (D - levels.astype(np.int64)))
    tgt = np.full(levels.shape, cfg.level_min, dtype=np.int64)
    for p in cfg.punctures:
        d2 = np.zeros(levels.shape, dtype=np.float64)
        parts = []
        for ax, pc in enumerate((p.x, p.y, p.z)):
            lo = cfg.xmin[ax] + anchors[:, ax].astype(np.float64) * unit
            hi = cfg.xmin[ax] + (anchors[:, ax] + side).astype(np.float64) * unit
            dd = np.maximum(np.maximum(lo - pc, 0.0), pc - hi)
            parts.append(dd * dd)
        d2 = (parts[0] + parts[1]) + parts[2]
        r2 = (cfg.rho * p.m) * (cfg.rho * p.m)
        j = np.zeros(levels.shape, dtype=np.int64)
        bound = np.full(levels.shape, r2, dtype=np.float64)
        for _ in range(64):
            far = d2 > bound
            if not far.any():
                break
            j[far] += 1
            bound[far] *= 4.0
        tgt = np.maximum(tgt, p.level - j)
    return tgt


def children(anchors: np.ndarray, levels: np.ndarray, D: int):
    """8 children of each octant, child c = x + 2y + 4z."""
    half = (np.int64(1) << (D - levels.astype(np.int64) - 1))
    out_a, out_l = [], []
    for c in range(8):
        off = np.stack([(c >> 0) & 1, (c >> 1) & 1, (c >> 2) & 1]).astype(np.int64)
        out_a.append(anchors + off[None, :] * half[:, None])
        out_l.append(levels + 1)
    return np.concatenate(out_a), np.concatenate(out_l)


def refine(cfg):
    """Top-down: an octant is split while its level is below its target."""
    D = cfg.max_depth
    leaves_a, leaves_l = [], []
    cur_a = np.zeros((1, 3), dtype=np.int64)
    cur_l = np.zeros(1, dtype=np.int64)
    while len(cur_l):
        tgt = target_levels(cur_a, cur_l, cfg)
        split = cur_l < tgt
        leaves_a.append(cur_a[~split])
        leaves_l.append(cur_l[~split])
        if split.any():
            cur_a, cur_l = children(cur_a[split], cur_l[split], D)
        else:
            break
    return np.concatenate(leaves_a), np.concatenate(leaves_l)


# ------------------------------------------------------------- point location

class Locator:
    """Leaf containing a depth-D cell, by binary search over Morton keys.

    Leaves of a complete linear octree partition the domain, so the leaf that
    contains cell c is the last leaf whose anchor key is <= key(c).
    """

    def __init__(self, anchors, levels, D, periodic):
        self.D = D
        self.n = 1 << D
        self.periodic = periodic
        self.anchors = anchors
        self.levels = levels
        self.keys = morton_key(anchors[:, 0], anchors[:, 1], anchors[:, 2], D)
        assert np.all(np.diff(self.keys) > 0), "leaves must be Morton sorted"

    def leaf_of_cell(self, cx, cy, cz):
        """Index of the leaf containing cell (cx,cy,cz); -1 if outside a
        non-periodic domain.  Periodic domains wrap."""
        cx = np.asarray(cx, dtype=np.int64)
        cy = np.asarray(cy, dtype=np.int64)
        cz = np.asarray(cz, dtype=np.int64)
        if self.periodic:
            cx, cy, cz = cx % self.n, cy % self.n, cz % self.n
            inside = np.ones(cx.shape, dtype=bool)
        else:
            inside = ((cx >= 0) & (cx < self.n) & (cy >= 0) & (cy < self.n)
                      & (cz >= 0) & (cz < self.n))
        k = morton_key(np.where(inside, cx, 0), np.where(inside, cy, 0),
                       np.where(inside, cz, 0), self.D)
        idx = np.searchsorted(self.keys, k, side="right") - 1
        return np.where(inside, idx, -1)


# ---------------------------------------------------------------- 2:1 balance

DIRS26 = np.array([(dx, dy, dz) for dz in (-1, 0, 1) for dy in (-1, 0, 1)
                   for dx in (-1, 0, 1) if (dx, dy, dz) != (0, 0, 0)], dtype=np.int64)


def balance(anchors, levels, D, periodic):
    """Minimal 2:1 vertex-balance closure.

    Repeat: for every leaf q of level L and each of the 26 directions d, look
    at the depth-D cell just outside q in direction d (a cell of q's
    same-level neighbour box N_d); if the leaf containing it has level < L-1
    it violates the balance with q and is split.  Stop when nothing splits.
    Any coarser leaf touching q contains a whole N_d, so these 26 probes see
    every violation.
    """
    anchors, levels = sort_morton(anchors, levels, D)
    while True:
        loc = Locator(anchors, levels, D, periodic)
        side = (np.int64(1) << (D - levels))
        mark = np.zeros(len(levels), dtype=bool)
        for d in DIRS26:
            c = []
            for ax in range(3):
                a = anchors[:, ax]
                c.append(np.where(d[ax] < 0, a - 1, np.where(d[ax] > 0, a + side, a)))
            nb = loc.leaf_of_cell(c[0], c[1], c[2])
            ok = nb >= 0
            viol = ok & (levels[np.where(ok, nb, 0)] < levels - 1)
            mark[nb[viol]] = True
        if not mark.any():
            return anchors, levels
        ca, cl = children(anchors[mark], levels[mark], D)
        anchors = np.concatenate([anchors[~mark], ca])
        levels = np.concatenate([levels[~mark], cl])
        anchors, levels = sort_morton(anchors, levels, D)


def build_octree(cfg):
    """refine -> balance -> Morton sort.  Returns (anchors int64 [N,3], levels int64 [N])."""
    a, l = refine(cfg)
    return balance(a, l, cfg.max_depth, cfg.periodic)


# --------------------------------------------------------------- validation

def is_complete(anchors, levels, D) -> bool:
    vol = np.sum((np.int64(1) << (3 * (D - levels))).astype(object))
    return int(vol) == (1 << (3 * D))


def touching(a1, l1, a2, l2, D, periodic):
    """Closed boxes of two octants intersect (and they are different octants)."""
    n = 1 << D
    s1 = 1 << (D - int(l1))
    s2 = 1 << (D - int(l2))
    for ax in range(3):
        lo1, hi1 = int(a1[ax]), int(a1[ax]) + s1
        lo2, hi2 = int(a2[ax]), int(a2[ax]) + s2
        if periodic:
            hit = any(lo1 <= hi2 + sh and lo2 + sh <= hi1 for sh in (-n, 0, n))
        else:
            hit = lo1 <= hi2 and lo2 <= hi1
        if not hit:
            return False
    return True


def is_balanced_bruteforce(anchors, levels, D, periodic) -> bool:
    """O(N^2) check of the 2:1 vertex balance — for tiny trees only."""
    N = len(levels)
    for i in range(N):
        for j in range(i + 1, N):
            if abs(int(levels[i]) - int(levels[j])) > 1 and touching(
                    anchors[i], levels[i], anchors[j], levels[j], D, periodic):
                return False
    return True
