"""ORACLE (test infrastructure only): grid points, DOFs, hanging points, zip
owners and padding (octant-to-patch) sources on a balanced linear octree.

Definitions (§III-C: each leaf has r^3 = 7^3 uniformly placed
points, "duplicate and hanging points are removed", patches are padded by
k = 3 points per direction; L184: O2N map; L241/L254: the octant-to-patch
neighbour map; readings R14-R17 in DESIGN.md):

* Node lattice: integer coordinates in units of (width/2^D)/6.  Node (i,j,k)
  of octant e (anchor a, side s = 2^(D-l)) is X = 6a + (i,j,k)*s, i..k in 0..6,
  local index n = i + 7j + 49k (x fastest).
* A point X is a DOF iff it lies on the node grid of EVERY leaf whose closed
  box contains it; otherwise it is hanging for the finer leaves.
* DOF numbering: octants in Morton order, nodes x-fastest, next id on first
  sight.  Since a DOF is a node of every leaf containing it, the first leaf
  that sees it is the lowest-index leaf containing it.
* Hanging source: the coarser leaf containing X, lowest Morton index on ties.
* Zip owner of a DOF: the COARSEST leaf containing it, lowest index on ties
  (reading R17, round 2: with the finest leaf as owner, the value of a node
  shared by a coarse and a fine leaf is updated from the fine leaf's
  stencil, whose padding is interpolated from the coarse leaf's values at
  that node, a feedback loop that makes moving-puncture runs blow up at
  every refinement interface the gauge pulse crosses; with the coarsest
  leaf the shared node is updated from the coarse stencil, which reads the
  fine side by injection: DESIGN.md §8b, profiles/r2_long_run_*).
* Padding source of patch point x of octant b: the finest leaf TOUCHING b whose
  closed box contains x, lowest index on ties; kind = copy (same level),
  inject (source finer), interp (source coarser); points outside a
  non-periodic domain are 'extrap'; a source reached through the periodic
  boundary carries the WRAP flag.

Containing leaves of a lattice point X are found by locating the 8 depth-D
cells floor((2X +- 1)/12) around it (oracle.octree.Locator).
"""
from __future__ import annotations

import numpy as np

from .octree import Locator, build_octree

R = 7            # points per octant edge
K = 3            # padding width
P13 = R + 2 * K  # patch edge, 13

KIND_SELF, KIND_COPY, KIND_INJECT, KIND_INTERP, KIND_EXTRAP = 0, 1, 2, 3, 4
KIND_WRAP = 8

_DIRS8 = np.array([(dx, dy, dz) for dz in (-1, 1) for dy in (-1, 1) for dx in (-1, 1)],
                  dtype=np.int64)


def _local_ijk():
    n = np.arange(R ** 3)
    return np.stack([n % R, (n // R) % R, n // (R * R)], axis=1)


def _patch_ijk():
    p = np.arange(P13 ** 3)
    return np.stack([p % P13, (p // P13) % P13, p // (P13 * P13)], axis=1)


class OracleMesh:
    """Balanced octree + all index maps, computed from the definitions above."""

    def __init__(self, cfg, anchors=None, levels=None):
        self.cfg = cfg
        self.D = cfg.max_depth
        self.periodic = cfg.periodic
        if anchors is None:
            anchors, levels = build_octree(cfg)
        self.anchors = np.asarray(anchors, dtype=np.int64)
        self.levels = np.asarray(levels, dtype=np.int64)
        self.n_oct = len(self.levels)
        self.side = (np.int64(1) << (self.D - self.levels))
        self.L = 6 * (1 << self.D)          # node-lattice extent
        self.loc = Locator(self.anchors, self.levels, self.D, self.periodic)
        if self.periodic:
            assert self.levels.min() >= 1
        self._dofs_done = False

    # ------------------------------------------------------------ geometry
    def h(self, e):
        """Grid spacing of octant e: width / (6 * 2^level)."""
        return self.cfg.width / (6.0 * (2.0 ** self.levels[e]))

    def node_X(self, e, ijk):
        """Lattice coordinates of local points ijk (int array [...,3]) of octants e."""
        e = np.asarray(e)
        return 6 * self.anchors[e] + ijk * self.side[e][..., None]

    def containing(self, X):
        """[M,8] leaf indices whose closed box contains lattice point X ([M,3]);
        entries are -1 (outside / duplicate-free not enforced)."""
        X = np.asarray(X, dtype=np.int64)
        out = np.empty((X.shape[0], 8), dtype=np.int64)
        for q, d in enumerate(_DIRS8):
            c = (2 * X + d[None, :]) // 12
            out[:, q] = self.loc.leaf_of_cell(c[:, 0], c[:, 1], c[:, 2])
        return out

    def _offset(self, X, c):
        """X - 6*a_c (periodic: taken modulo the lattice extent into [0, 6 s_c])."""
        off = X - 6 * self.anchors[c]
        if self.periodic:
            off = off % self.L
        return off

    def on_grid(self, X, c):
        off = self._offset(X, c)
        s = self.side[c][:, None]
        return np.all(off % s == 0, axis=1)

    # ----------------------------------------------------- DOFs / hanging
    def build_dofs(self, chunk=4096):
        """O2N (DOF id or -1), hanging sources and zip owners."""
        if self._dofs_done:
            return
        N = self.n_oct
        ijk = _local_ijk()
        is_bdy = np.any((ijk == 0) | (ijk == R - 1), axis=1)
        bidx = np.nonzero(is_bdy)[0]
        nb = len(bidx)
        is_dof = np.ones((N, R ** 3), dtype=bool)
        first = np.repeat(np.arange(N)[:, None], R ** 3, axis=1)   # lowest containing leaf
        hang_src = np.full((N, R ** 3), -1, dtype=np.int64)
        owner = np.repeat(np.arange(N)[:, None], R ** 3, axis=1)   # zip owner leaf
        for e0 in range(0, N, chunk):
            e1 = min(N, e0 + chunk)
            ee = np.repeat(np.arange(e0, e1), nb)
            X = self.node_X(ee, np.tile(ijk[bidx], (e1 - e0, 1)))
            cont = self.containing(X)
            M = len(ee)
            dof = np.ones(M, dtype=bool)
            fst = np.full(M, np.iinfo(np.int64).max)
            hs = np.full(M, np.iinfo(np.int64).max)
            own = np.full(M, -1, dtype=np.int64)
            own_lvl = np.full(M, np.iinfo(np.int64).max, dtype=np.int64)
            for q in range(8):
                c = cont[:, q]
                ok = c >= 0
                cc = np.where(ok, c, 0)
                og = self.on_grid(X, cc)
                dof &= ~ok | og
                fst = np.where(ok, np.minimum(fst, cc), fst)
                coarser = ok & (self.levels[cc] < self.levels[ee])
                hs = np.where(coarser, np.minimum(hs, cc), hs)
                lv = self.levels[cc]
                better = ok & ((lv < own_lvl) | ((lv == own_lvl) & (cc < own)))
                own = np.where(better, cc, own)
                own_lvl = np.where(better, lv, own_lvl)
            sl = (slice(e0, e1), bidx)
            is_dof[sl] = dof.reshape(e1 - e0, nb)
            first[sl] = fst.reshape(e1 - e0, nb)
            hang_src[sl] = np.where(dof, -1, hs).reshape(e1 - e0, nb)
            owner[sl] = own.reshape(e1 - e0, nb)
        # numbering: first-sight nodes in (octant, x-fastest node) order
        new = is_dof & (first == np.arange(N)[:, None])
        o2n = np.full((N, R ** 3), -1, dtype=np.int64)
        o2n[new] = np.arange(int(new.sum()))
        self.n_dof = int(new.sum())
        # other DOF nodes take the id the first leaf gave them
        rest = is_dof & ~new
        ee, nn = np.nonzero(rest)
        X = self.node_X(ee, ijk[nn])
        f = first[ee, nn]
        loc_f = self._offset(X, f) // self.side[f][:, None]
        nf = loc_f[:, 0] + R * loc_f[:, 1] + R * R * loc_f[:, 2]
        assert np.all(o2n[f, nf] >= 0)
        o2n[ee, nn] = o2n[f, nf]
        self.o2n = o2n
        self.is_dof = is_dof
        self.hang_src = hang_src
        # zip owners: (leaf, local index) for each DOF id
        zo_leaf = np.full(self.n_dof, -1, dtype=np.int64)
        zo_node = np.full(self.n_dof, -1, dtype=np.int64)
        ee, nn = np.nonzero(is_dof & (owner == np.arange(N)[:, None]))
        zo_leaf[o2n[ee, nn]] = ee
        zo_node[o2n[ee, nn]] = nn
        assert np.all(zo_leaf >= 0)
        self.zip_leaf, self.zip_node = zo_leaf, zo_node
        self._dofs_done = True

    def dof_lattice(self):
        """Lattice coordinates [n_dof, 3] of the DOFs (X = 6 anchor + i side)."""
        self.build_dofs()
        return self.node_X(self.zip_leaf, _local_ijk()[self.zip_node])

    def dof_coords(self):
        """Physical coordinates [3, n_dof] of the DOFs."""
        self.build_dofs()
        X = self.node_X(self.zip_leaf, _local_ijk()[self.zip_node])
        unit = self.cfg.width / self.L
        return np.stack([self.cfg.xmin[a] + X[:, a] * unit for a in range(3)])

    def hanging_table(self):
        """Rows (octant, node, source leaf) of every hanging point, sorted."""
        self.build_dofs()
        ee, nn = np.nonzero(~self.is_dof)
        return np.stack([ee, nn, self.hang_src[ee, nn]], axis=1)

    # ---------------------------------------------------- padding sources
    def padding_sources(self, octs=None):
        """(src [n,2197] int64, kind [n,2197] uint8) for octants `octs`."""
        octs = np.arange(self.n_oct) if octs is None else np.asarray(octs, dtype=np.int64)
        pijk = _patch_ijk()
        interior = np.all((pijk >= K) & (pijk < K + R), axis=1)
        pad = np.nonzero(~interior)[0]
        n = len(octs)
        src = np.repeat(octs[:, None], P13 ** 3, axis=1).astype(np.int64)
        kind = np.zeros((n, P13 ** 3), dtype=np.uint8)
        bb = np.repeat(octs, len(pad))
        X = 6 * self.anchors[bb] + (np.tile(pijk[pad], (n, 1)) - K) * self.side[bb][:, None]
        M = len(bb)
        if self.periodic:
            Xw = X % self.L
            outside = np.zeros(M, dtype=bool)
        else:
            Xw = X
            outside = np.any((X < 0) | (X > self.L), axis=1)
        cont = self.containing(np.where(outside[:, None], 0, Xw))
        best = np.full(M, -1, dtype=np.int64)
        best_l = np.full(M, -1, dtype=np.int64)
        best_w = np.zeros(M, dtype=bool)
        lo_b = 6 * self.anchors[bb]
        hi_b = lo_b + 6 * self.side[bb][:, None]
        for q in range(8):
            c = cont[:, q]
            ok = (c >= 0) & ~outside
            cc = np.where(ok, c, 0)
            lo_c = 6 * self.anchors[cc]
            hi_c = lo_c + 6 * self.side[cc][:, None]
            # shift of the candidate box (multiple of L) that puts X inside it
            sh = np.zeros_like(X)
            if self.periodic:
                for s in (-self.L, self.L):
                    fit = (lo_c + s <= X) & (X <= hi_c + s)
                    sh = np.where(fit & ~((lo_c <= X) & (X <= hi_c)), s, sh)
            lo_s, hi_s = lo_c + sh, hi_c + sh
            inside = np.all((lo_s <= X) & (X <= hi_s), axis=1)
            touch = np.all((lo_s <= hi_b) & (lo_b <= hi_s), axis=1)
            cand = ok & inside & touch
            lv = self.levels[cc]
            better = cand & ((lv > best_l) | ((lv == best_l) & (cc < best)))
            best = np.where(better, cc, best)
            best_l = np.where(better, lv, best_l)
            best_w = np.where(better, np.any(sh != 0, axis=1), best_w)
        assert np.all((best >= 0) | outside), "uncovered padding point"
        lb = self.levels[bb]
        kd = np.where(best_l == lb, KIND_COPY,
                      np.where(best_l > lb, KIND_INJECT, KIND_INTERP)).astype(np.uint8)
        kd = np.where(best_w, kd | KIND_WRAP, kd).astype(np.uint8)
        kd = np.where(outside, KIND_EXTRAP, kd).astype(np.uint8)
        best = np.where(outside, -1, best)
        src[:, pad] = best.reshape(n, len(pad))
        kind[:, pad] = kd.reshape(n, len(pad))
        return src, kind
