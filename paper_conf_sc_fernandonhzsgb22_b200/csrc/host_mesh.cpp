// Host-side octree + maps. See host_mesh.hpp for the contract.
// Compiled with -ffp-contract=off: the refinement rule's floating point must
// round exactly as written (DESIGN.md R-O1).
#include "host_mesh.hpp"

#include <omp.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <unordered_map>
#include <unordered_set>

namespace dgr {

static inline uint64_t spread3(uint64_t v) {
  v &= 0x1fffffULL;
  v = (v | (v << 32)) & 0x1f00000000ffffULL;
  v = (v | (v << 16)) & 0x1f0000ff0000ffULL;
  v = (v | (v << 8)) & 0x100f00f00f00f00fULL;
  v = (v | (v << 4)) & 0x10c30c30c30c30c3ULL;
  v = (v | (v << 2)) & 0x1249249249249249ULL;
  return v;
}

uint64_t morton(int64_t x, int64_t y, int64_t z, int /*D*/) {
  return spread3(uint64_t(x)) | (spread3(uint64_t(y)) << 1) | (spread3(uint64_t(z)) << 2);
}

static inline uint64_t pack(int64_t x, int64_t y, int64_t z) {
  return uint64_t(x) | (uint64_t(y) << 21) | (uint64_t(z) << 42);
}

// ------------------------------------------------------------ refinement

namespace {
struct Refiner {
  double xmin[3], width, unit, rho;
  int D, level_min;
  std::vector<PunctureDesc> p;

  int target(const int64_t a[3], int l) const {
    const int64_t s = int64_t(1) << (D - l);
    int t = level_min;
    for (const auto& q : p) {
      const double pc[3] = {q.x, q.y, q.z};
      double part[3];
      for (int ax = 0; ax < 3; ++ax) {
        const double lo = xmin[ax] + double(a[ax]) * unit;
        const double hi = xmin[ax] + double(a[ax] + s) * unit;
        const double dd = std::max(std::max(lo - pc[ax], 0.0), pc[ax] - hi);
        part[ax] = dd * dd;
      }
      const double d2 = (part[0] + part[1]) + part[2];
      const double r2 = (rho * q.m) * (rho * q.m);
      double bound = r2;
      int j = 0;
      while (d2 > bound && j < 64) {
        ++j;
        bound *= 4.0;
      }
      t = std::max(t, q.level - j);
    }
    return t;
  }
};
}  // namespace

std::vector<Oct> balance_internal(std::vector<std::unordered_set<uint64_t>>& I, int D,
                                  bool periodic);

std::vector<Oct> build_octree(const double xmin[3], double width, int D, bool periodic,
                              int level_min, const std::vector<PunctureDesc>& punct,
                              double rho) {
  Refiner rf;
  for (int i = 0; i < 3; ++i) rf.xmin[i] = xmin[i];
  rf.width = width;
  rf.unit = std::ldexp(width, -D);
  rf.rho = rho;
  rf.D = D;
  rf.level_min = level_min;
  rf.p = punct;
  // internal-node sets per level, from the refinement rule (top-down)
  std::vector<std::unordered_set<uint64_t>> I(D + 1);
  {
    std::vector<Oct> cur{{{0, 0, 0}, 0}};
    while (!cur.empty()) {
      std::vector<Oct> nxt;
      for (const Oct& o : cur) {
        if (o.l < D && o.l < rf.target(o.a, o.l)) {
          I[o.l].insert(pack(o.a[0], o.a[1], o.a[2]));
          const int64_t h = int64_t(1) << (D - o.l - 1);
          for (int c = 0; c < 8; ++c)
            nxt.push_back({{o.a[0] + (c & 1) * h, o.a[1] + ((c >> 1) & 1) * h,
                            o.a[2] + ((c >> 2) & 1) * h},
                           o.l + 1});
        }
      }
      cur.swap(nxt);
    }
  }
  return balance_internal(I, D, periodic);
}

// Minimal 2:1 vertex-balance closure of the tree whose internal nodes per
// level are I, then its leaves in Morton order (shared by the builder and the
// regrid).
std::vector<Oct> balance_internal(std::vector<std::unordered_set<uint64_t>>& I, int D,
                                  bool periodic) {
  int maxl = 0;
  for (int l = 0; l <= D; ++l)
    if (!I[l].empty()) maxl = l + 1;
  // ripple balance, finest level first: every present node q at level L
  // requires the level-(L-1) node containing each same-level neighbour box to
  // be present, i.e. its parent (level L-2) to be internal.
  const int64_t n = int64_t(1) << D;
  auto ensure = [&](int64_t x, int64_t y, int64_t z, int l) {
    while (l >= 0) {
      const int64_t s = int64_t(1) << (D - l);
      x = (x / s) * s;
      y = (y / s) * s;
      z = (z / s) * s;
      if (!I[l].insert(pack(x, y, z)).second) return;
      --l;
    }
  };
  for (int Lv = maxl; Lv >= 2; --Lv) {
    std::vector<uint64_t> parents(I[Lv - 1].begin(), I[Lv - 1].end());
    const int64_t s = int64_t(1) << (D - Lv);
    for (uint64_t pk : parents) {
      const int64_t px = pk & 0x1fffff, py = (pk >> 21) & 0x1fffff, pz = (pk >> 42) & 0x1fffff;
      for (int c = 0; c < 8; ++c) {
        const int64_t q[3] = {px + (c & 1) * s, py + ((c >> 1) & 1) * s, pz + ((c >> 2) & 1) * s};
        for (int dz = -1; dz <= 1; ++dz)
          for (int dy = -1; dy <= 1; ++dy)
            for (int dx = -1; dx <= 1; ++dx) {
              if (!dx && !dy && !dz) continue;
              int64_t nb[3] = {q[0] + dx * s, q[1] + dy * s, q[2] + dz * s};
              bool ok = true;
              for (int k = 0; k < 3; ++k) {
                if (nb[k] < 0 || nb[k] >= n) {
                  if (periodic)
                    nb[k] = ((nb[k] % n) + n) % n;
                  else
                    ok = false;
                }
              }
              if (ok) ensure(nb[0], nb[1], nb[2], Lv - 2);
            }
      }
    }
  }
  // leaves by DFS in child order c = x + 2y + 4z == Morton order
  std::vector<Oct> out;
  std::vector<Oct> stack{{{0, 0, 0}, 0}};
  while (!stack.empty()) {
    Oct o = stack.back();
    stack.pop_back();
    if (o.l < D && I[o.l].count(pack(o.a[0], o.a[1], o.a[2]))) {
      const int64_t h = int64_t(1) << (D - o.l - 1);
      for (int c = 7; c >= 0; --c)
        stack.push_back({{o.a[0] + (c & 1) * h, o.a[1] + ((c >> 1) & 1) * h,
                          o.a[2] + ((c >> 2) & 1) * h},
                         o.l + 1});
    } else {
      out.push_back(o);
    }
  }
  return out;
}

std::vector<Oct> regrid_leaves(const std::vector<Oct>& leaves, const double* w, double eps_refine,
                              double eps_coarsen, int level_min, int level_max, int D,
                              bool periodic) {
  // reading R31: split leaves above eps_refine (level < level_max),
  // merge complete families of 8 sibling leaves all below eps_coarsen (level >
  // level_min, none split), then the minimal balance closure
  const size_t N = leaves.size();
  std::vector<uint8_t> split(N, 0), merged(N, 0);
  for (size_t e = 0; e < N; ++e) split[e] = w[e] > eps_refine && leaves[e].l < level_max;
  std::vector<Oct> nl;
  for (size_t e = 0; e < N;) {
    const Oct& o = leaves[e];
    const int64_t s = int64_t(1) << (D - o.l);
    // a family starts at child 0 of its parent: 8 consecutive same-level
    // leaves (Morton order) with one parent
    bool fam = o.l > level_min && e + 8 <= N && o.l > 0 &&
               (o.a[0] & (2 * s - 1)) == 0 && (o.a[1] & (2 * s - 1)) == 0 &&
               (o.a[2] & (2 * s - 1)) == 0;
    for (size_t c = 0; fam && c < 8; ++c) {
      const Oct& q = leaves[e + c];
      fam = q.l == o.l && q.a[0] == o.a[0] + int64_t(c & 1) * s &&
            q.a[1] == o.a[1] + int64_t((c >> 1) & 1) * s &&
            q.a[2] == o.a[2] + int64_t((c >> 2) & 1) * s && !split[e + c] &&
            w[e + c] < eps_coarsen;
    }
    if (fam) {
      nl.push_back({{o.a[0], o.a[1], o.a[2]}, o.l - 1});
      e += 8;
      continue;
    }
    if (split[e]) {
      const int64_t h = s / 2;
      for (int c = 0; c < 8; ++c)
        nl.push_back({{o.a[0] + (c & 1) * h, o.a[1] + ((c >> 1) & 1) * h,
                       o.a[2] + ((c >> 2) & 1) * h}, o.l + 1});
    } else {
      nl.push_back(o);
    }
    ++e;
  }
  std::vector<std::unordered_set<uint64_t>> I(D + 1);
  for (const Oct& o : nl)
    for (int l = 0; l < o.l; ++l) {
      const int64_t s = int64_t(1) << (D - l);
      I[l].insert(pack((o.a[0] / s) * s, (o.a[1] / s) * s, (o.a[2] / s) * s));
    }
  return balance_internal(I, D, periodic);
}

// --------------------------------------------------------------- HostMesh

int32_t HostMesh::locate(int64_t cx, int64_t cy, int64_t cz) const {
  const int64_t n = int64_t(1) << D;
  if (periodic) {
    cx = ((cx % n) + n) % n;
    cy = ((cy % n) + n) % n;
    cz = ((cz % n) + n) % n;
  } else if (cx < 0 || cy < 0 || cz < 0 || cx >= n || cy >= n || cz >= n) {
    return -1;
  }
  const uint64_t k = morton(cx, cy, cz, D);
  auto it = std::upper_bound(key.begin(), key.end(), k);
  return int32_t(it - key.begin()) - 1;
}

void HostMesh::validate() {
  const int64_t N = int64_t(oct.size());
  if (N == 0) throw BuildError{-2, "empty octant list"};
  key.resize(N);
  const int64_t n = int64_t(1) << D;
  for (int64_t i = 0; i < N; ++i) {
    const Oct& o = oct[i];
    if (o.l < 0 || o.l > D) throw BuildError{-2, "octant level out of range"};
    const int64_t s = int64_t(1) << (D - o.l);
    for (int k = 0; k < 3; ++k)
      if (o.a[k] < 0 || o.a[k] + s > n || o.a[k] % s)
        throw BuildError{-2, "octant anchor misaligned or outside the domain"};
    key[i] = morton(o.a[0], o.a[1], o.a[2], D);
  }
  // sorted, contiguous and complete: key_{i+1} = key_i + 8^(D - l_i)
  uint64_t expect = 0;
  for (int64_t i = 0; i < N; ++i) {
    if (key[i] != expect)
      throw BuildError{-2, "octants not sorted / overlapping / incomplete at index " +
                               std::to_string(i)};
    expect += uint64_t(1) << (3 * (D - oct[i].l));
  }
  if (expect != (uint64_t(1) << (3 * D))) throw BuildError{-2, "octants do not cover the domain"};
  // 2:1 vertex balance: the leaf holding the cell just outside q in each of
  // the 26 directions has level >= level(q) - 1
  int bad = 0;
#pragma omp parallel for reduction(+ : bad) schedule(static)
  for (int64_t i = 0; i < N; ++i) {
    const Oct& q = oct[i];
    const int64_t s = int64_t(1) << (D - q.l);
    for (int d = 0; d < 27; ++d) {
      const int dx = d % 3 - 1, dy = (d / 3) % 3 - 1, dz = d / 9 - 1;
      if (!dx && !dy && !dz) continue;
      const int64_t c[3] = {dx < 0 ? q.a[0] - 1 : (dx > 0 ? q.a[0] + s : q.a[0]),
                            dy < 0 ? q.a[1] - 1 : (dy > 0 ? q.a[1] + s : q.a[1]),
                            dz < 0 ? q.a[2] - 1 : (dz > 0 ? q.a[2] + s : q.a[2])};
      const int32_t nb = locate(c[0], c[1], c[2]);
      if (nb >= 0 && oct[nb].l < q.l - 1) ++bad;
    }
  }
  if (bad) throw BuildError{-2, "octree is not 2:1 vertex balanced"};
  level_min = 1 << 30;
  level_max = 0;
  for (const Oct& o : oct) {
    level_min = std::min(level_min, o.l);
    level_max = std::max(level_max, o.l);
  }
  if (periodic && level_min < 1) throw BuildError{-2, "periodic meshes need level >= 1"};
}

// Touching leaves of every leaf: probe the same-level neighbour box N_d in
// each of the 26 directions; a leaf at the same or a coarser level contains
// all of N_d; finer leaves (exactly one level finer under 2:1 balance) are the
// children of N_d adjacent to the octant.
void HostMesh::build_touch() {
  const int64_t N = int64_t(oct.size());
  const int64_t n = int64_t(1) << D;
  touch.assign(N, {});
  int bad = 0;
#pragma omp parallel for schedule(dynamic, 256) reduction(+ : bad)
  for (int64_t e = 0; e < N; ++e) {
    const Oct& q = oct[e];
    const int64_t s = int64_t(1) << (D - q.l);
    std::vector<Touch>& out = touch[e];
    auto add = [&](int32_t c, const int64_t sh[3]) {
      for (const Touch& t : out)
        if (t.leaf == c && t.sh[0] == sh[0] && t.sh[1] == sh[1] && t.sh[2] == sh[2]) return;
      out.push_back({c, {sh[0], sh[1], sh[2]}});
    };
    for (int d = 0; d < 27; ++d) {
      const int dd[3] = {d % 3 - 1, (d / 3) % 3 - 1, d / 9 - 1};
      if (!dd[0] && !dd[1] && !dd[2]) continue;
      int64_t nb[3], sh[3];
      bool ok = true;
      for (int k = 0; k < 3; ++k) {
        const int64_t raw = q.a[k] + dd[k] * s;
        int64_t w = raw;
        if (raw < 0 || raw >= n) {
          if (!periodic) ok = false;
          w = ((raw % n) + n) % n;
        }
        nb[k] = w;
        sh[k] = 6 * (raw - w);  // node-lattice shift that moves the leaf next to q
      }
      if (!ok) continue;
      const int32_t c = locate(nb[0], nb[1], nb[2]);
      if (oct[c].l <= q.l) {
        // coarser/same: the containing leaf's anchor may differ from nb, but
        // the shift is the same multiple of the domain
        add(c, sh);
      } else {
        const int64_t h = s / 2;
        for (int ch = 0; ch < 8; ++ch) {
          const int cb[3] = {ch & 1, (ch >> 1) & 1, (ch >> 2) & 1};
          bool adj = true;
          for (int k = 0; k < 3; ++k)
            if ((dd[k] < 0 && cb[k] != 1) || (dd[k] > 0 && cb[k] != 0)) adj = false;
          if (!adj) continue;
          const int32_t cc = locate(nb[0] + cb[0] * h, nb[1] + cb[1] * h, nb[2] + cb[2] * h);
          if (oct[cc].l != q.l + 1) ++bad;
          add(cc, sh);
        }
      }
    }
    if (int(out.size()) > NBR_MAX) ++bad;
  }
  if (bad) throw BuildError{-2, "inconsistent neighbourhood (balance violated?)"};
}

namespace {
struct NodeInfo {
  int8_t kind;       // 0 new DOF, 1 DOF seen first elsewhere, 2 hanging
  bool own;          // this leaf is the zip owner
  int32_t ref_leaf;  // kind 1: first leaf; kind 2: hanging source
  int16_t ref_node;  // kind 1: local node index in ref_leaf
  uint8_t t2[3];     // kind 2: half-grid coordinates in the source
};
}  // namespace

// DOF / hanging classification (R14-R17): X is a DOF iff it lies on
// the node grid of every leaf whose closed box contains it.
void HostMesh::classify_nodes() {
  const int64_t N = int64_t(oct.size());

  std::vector<NodeInfo> info(size_t(N) * NPT);
  std::vector<int32_t> n_new(N, 0);
  int bad = 0;
#pragma omp parallel for schedule(dynamic, 64) reduction(+ : bad)
  for (int64_t e = 0; e < N; ++e) {
    const Oct& q = oct[e];
    const int64_t s = side(int32_t(e));
    int cnt = 0;
    for (int node = 0; node < NPT; ++node) {
      const int ijk[3] = {node % 7, (node / 7) % 7, node / 49};
      NodeInfo& ni = info[size_t(e) * NPT + node];
      const bool bdy = ijk[0] == 0 || ijk[0] == 6 || ijk[1] == 0 || ijk[1] == 6 ||
                       ijk[2] == 0 || ijk[2] == 6;
      if (!bdy) {
        ni = {0, true, int32_t(e), int16_t(node), {0, 0, 0}};
        ++cnt;
        continue;
      }
      int64_t X[3];
      for (int k = 0; k < 3; ++k) X[k] = 6 * q.a[k] + ijk[k] * s;
      bool dof = true;
      int32_t first = int32_t(e);
      int64_t first_sh[3] = {0, 0, 0};
      int32_t hsrc = -1;
      int64_t hsh[3] = {0, 0, 0};
      int32_t own = int32_t(e);
      int own_l = q.l;
      for (const Touch& t : touch[e]) {
        const Oct& c = oct[t.leaf];
        const int64_t sc = side(t.leaf);
        bool in = true;
        for (int k = 0; k < 3; ++k) {
          const int64_t lo = 6 * c.a[k] + t.sh[k];
          if (X[k] < lo || X[k] > lo + 6 * sc) in = false;
        }
        if (!in) continue;
        bool on = true;
        for (int k = 0; k < 3; ++k)
          if ((X[k] - t.sh[k] - 6 * c.a[k]) % sc) on = false;
        if (!on) dof = false;
        if (t.leaf < first) {
          first = t.leaf;
          std::memcpy(first_sh, t.sh, sizeof(first_sh));
        }
        if (c.l < q.l && (hsrc < 0 || t.leaf < hsrc)) {
          hsrc = t.leaf;
          std::memcpy(hsh, t.sh, sizeof(hsh));
        }
        // zip owner (reading R17): the coarsest containing leaf, lowest index
        // on ties — a shared coarse/fine node is updated from the coarse
        // stencil (the finest-owner rule feeds the coarse->fine padding
        // interpolation back into the node and is unstable)
        if (c.l < own_l || (c.l == own_l && t.leaf < own)) {
          own = t.leaf;
          own_l = c.l;
        }
      }
      if (dof) {
        if (first == int32_t(e)) {
          ni = {0, own == int32_t(e), int32_t(e), int16_t(node), {0, 0, 0}};
          ++cnt;
        } else {
          const int64_t sf = side(first);
          int loc[3];
          for (int k = 0; k < 3; ++k)
            loc[k] = int((X[k] - first_sh[k] - 6 * oct[first].a[k]) / sf);
          ni = {1, own == int32_t(e), first, int16_t(loc[0] + 7 * loc[1] + 49 * loc[2]), {0, 0, 0}};
        }
      } else {
        if (hsrc < 0) {
          ++bad;
          continue;
        }
        const int64_t sc = side(hsrc);
        uint8_t t2[3];
        for (int k = 0; k < 3; ++k) {
          const int64_t num = 2 * (X[k] - hsh[k] - 6 * oct[hsrc].a[k]);
          if (num % sc || num / sc < 0 || num / sc > 12) ++bad;
          t2[k] = uint8_t(num / sc);
        }
        ni = {2, false, hsrc, 0, {t2[0], t2[1], t2[2]}};
      }
    }
    n_new[e] = cnt;
  }
  if (bad) throw BuildError{-2, "node classification failed (hanging point without coarser source)"};
  // first-sight numbering
  std::vector<int64_t> base(N + 1, 0);
  for (int64_t e = 0; e < N; ++e) base[e + 1] = base[e] + n_new[e];
  n_dof = base[N];
  if (n_dof > INT32_MAX) throw BuildError{-1, "too many DOFs for int32 ids"};
  o2n.assign(size_t(N) * NPT, -1);
  hang.assign(size_t(N) * NPT, HangRef{-1, {0, 0, 0}});
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < N; ++e) {
    int64_t id = base[e];
    for (int node = 0; node < NPT; ++node)
      if (info[size_t(e) * NPT + node].kind == 0) o2n[size_t(e) * NPT + node] = int32_t(id++);
  }
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < N; ++e) {
    for (int node = 0; node < NPT; ++node) {
      const NodeInfo& ni = info[size_t(e) * NPT + node];
      if (ni.kind == 1) {
        o2n[size_t(e) * NPT + node] = o2n[size_t(ni.ref_leaf) * NPT + ni.ref_node];
      } else if (ni.kind == 2) {
        hang[size_t(e) * NPT + node] = HangRef{ni.ref_leaf, {ni.t2[0], ni.t2[1], ni.t2[2]}};
      }
    }
  }
  zip_leaf.assign(n_dof, -1);
  zip_node.assign(n_dof, -1);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < N; ++e)
    for (int node = 0; node < NPT; ++node) {
      const NodeInfo& ni = info[size_t(e) * NPT + node];
      if (ni.kind != 2 && ni.own) {
        const int32_t id = o2n[size_t(e) * NPT + node];
        zip_leaf[id] = int32_t(e);
        zip_node[id] = node;
      }
    }
  for (int64_t d = 0; d < n_dof; ++d)
    if (zip_leaf[d] < 0) throw BuildError{-2, "DOF without zip owner"};
}

// Morton-contiguous partition: rank r owns leaves [N r / R, N (r+1) / R).
// Ghost octants: padding sources of owned octants, closed under hanging sources.
// Owned DOFs: zip owner is owned. Ghost DOFs: every other DOF referenced by a
// local (owned or ghost) octant, grouped by owning rank, sorted by global id.
void HostMesh::partition() {
  const int64_t N = int64_t(oct.size());
  oct_begin = N * rank / nranks;
  oct_end = N * (rank + 1) / nranks;
  n_owned_oct = oct_end - oct_begin;
  auto owner_of_oct = [&](int64_t g) {
    // inverse of the floor partition
    int r = int(((g + 1) * nranks - 1) / N);
    while (r > 0 && N * r / nranks > g) --r;
    while (r + 1 < nranks && N * (r + 1) / nranks <= g) ++r;
    return r;
  };
  g2l_oct.assign(N, -1);
  local_oct.clear();
  for (int64_t g = oct_begin; g < oct_end; ++g) {
    g2l_oct[g] = int32_t(local_oct.size());
    local_oct.push_back(int32_t(g));
  }
  if (nranks > 1) {
    std::vector<char> need(N, 0);
    for (int64_t g = oct_begin; g < oct_end; ++g)
      for (const Touch& t : touch[g]) need[t.leaf] = 1;
    // hanging closure over needed octants (sources are coarser: iterate to a fixed point)
    bool changed = true;
    while (changed) {
      changed = false;
      for (int64_t g = 0; g < N; ++g) {
        if (!(need[g] || (g >= oct_begin && g < oct_end))) continue;
        for (int node = 0; node < NPT; ++node) {
          const int32_t src = hang[size_t(g) * NPT + node].src;
          if (src >= 0 && !need[src] && !(src >= oct_begin && src < oct_end)) {
            need[src] = 1;
            changed = true;
          }
        }
      }
    }
    for (int64_t g = 0; g < N; ++g)
      if (need[g] && !(g >= oct_begin && g < oct_end)) {
        g2l_oct[g] = int32_t(local_oct.size());
        local_oct.push_back(int32_t(g));
      }
  }
  n_ghost_oct = int64_t(local_oct.size()) - n_owned_oct;
  // DOF owner ranks
  dof_owner_rank.assign(n_dof, 0);
  if (nranks > 1)
    for (int64_t d = 0; d < n_dof; ++d) dof_owner_rank[d] = owner_of_oct(zip_leaf[d]);
  // owned DOFs in global-id order
  std::unordered_map<int64_t, int32_t> g2l_dof;
  dof_gid.clear();
  for (int64_t d = 0; d < n_dof; ++d)
    if (dof_owner_rank[d] == rank) {
      g2l_dof[d] = int32_t(dof_gid.size());
      dof_gid.push_back(d);
    }
  n_owned_dof = int64_t(dof_gid.size());
  // ghost DOFs referenced by local octants
  std::vector<std::vector<int64_t>> ghost_by_rank(nranks);
  {
    std::unordered_set<int64_t> seen;
    for (int32_t g : local_oct)
      for (int node = 0; node < NPT; ++node) {
        const int32_t id = o2n[size_t(g) * NPT + node];
        if (id >= 0 && dof_owner_rank[id] != rank && seen.insert(id).second)
          ghost_by_rank[dof_owner_rank[id]].push_back(id);
      }
  }
  recv_counts.assign(nranks, 0);
  for (int r = 0; r < nranks; ++r) {
    auto& v = ghost_by_rank[r];
    std::sort(v.begin(), v.end());
    recv_counts[r] = int64_t(v.size());
    for (int64_t id : v) {
      g2l_dof[id] = int32_t(dof_gid.size());
      dof_gid.push_back(id);
    }
  }
  n_ghost_dof = int64_t(dof_gid.size()) - n_owned_dof;
  // local O2N
  const int64_t nl = int64_t(local_oct.size());
  o2n_local.assign(size_t(nl) * NPT, -1);
  for (int64_t l = 0; l < nl; ++l)
    for (int node = 0; node < NPT; ++node) {
      const int32_t id = o2n[size_t(local_oct[l]) * NPT + node];
      if (id >= 0) o2n_local[size_t(l) * NPT + node] = g2l_dof.at(id);
    }
  // send lists: what every peer needs from us (peers build the same global maps)
  send_counts.assign(nranks, 0);
  send_list.clear();
  if (nranks > 1) {
    for (int peer = 0; peer < nranks; ++peer) {
      if (peer == rank) continue;
      const int64_t pb = N * peer / nranks, pe = N * (peer + 1) / nranks;
      std::vector<char> pneed(N, 0);
      for (int64_t g = pb; g < pe; ++g) {
        pneed[g] = 1;
        for (const Touch& t : touch[g]) pneed[t.leaf] = 1;
      }
      bool changed = true;
      while (changed) {
        changed = false;
        for (int64_t g = 0; g < N; ++g) {
          if (!pneed[g]) continue;
          for (int node = 0; node < NPT; ++node) {
            const int32_t src = hang[size_t(g) * NPT + node].src;
            if (src >= 0 && !pneed[src]) {
              pneed[src] = 1;
              changed = true;
            }
          }
        }
      }
      std::vector<int64_t> ids;
      std::unordered_set<int64_t> seen;
      for (int64_t g = 0; g < N; ++g) {
        if (!pneed[g]) continue;
        for (int node = 0; node < NPT; ++node) {
          const int32_t id = o2n[size_t(g) * NPT + node];
          if (id >= 0 && dof_owner_rank[id] == rank && owner_of_oct(zip_leaf[id]) == rank) {
            // peer needs it unless it owns it (it does not: we own it)
            if (seen.insert(id).second) ids.push_back(id);
          }
        }
      }
      std::sort(ids.begin(), ids.end());
      send_counts[peer] = int64_t(ids.size());
      for (int64_t id : ids) send_list.push_back(g2l_dof.at(id));
    }
  }
  // zip: owned DOF -> local octant * 343 + node
  zip_local.assign(n_owned_dof, 0);
  for (int64_t l = 0; l < n_owned_dof; ++l) {
    const int64_t id = dof_gid[l];
    zip_local[l] = g2l_oct[zip_leaf[id]] * NPT + zip_node[id];
  }
  // hanging rows over local octants, sorted by (level, local octant, node)
  hang_rows.clear();
  for (int64_t l = 0; l < nl; ++l) {
    const int32_t g = local_oct[l];
    for (int node = 0; node < NPT; ++node) {
      const HangRef& h = hang[size_t(g) * NPT + node];
      if (h.src < 0) continue;
      if (g2l_oct[h.src] < 0) throw BuildError{-2, "hanging source missing from ghost layer"};
      HangRow r;
      r.e_local = int32_t(l);
      r.node = node;
      r.src_local = g2l_oct[h.src];
      std::memcpy(r.t2, h.t2, 3);
      r.level = oct[g].l;
      r.e_global = g;
      r.src_global = h.src;
      hang_rows.push_back(r);
    }
  }
  std::stable_sort(hang_rows.begin(), hang_rows.end(),
                   [](const HangRow& a, const HangRow& b) { return a.level < b.level; });
  // dependency depth (reading R14): a row whose interpolation stencil on its
  // source octant touches only DOF nodes has depth 0, otherwise 1 + the
  // deepest hanging node it reads.  Rows of equal depth are independent, so
  // the device resolves one depth per launch (typically 2-3 instead of one
  // launch per level).  Level order guarantees sources are visited first.
  std::vector<int32_t> depth_of(size_t(nl) * NPT, -1);
  for (HangRow& r : hang_rows) {
    int d = 0;
    const int nx = (r.t2[0] & 1) ? 7 : 1, ny = (r.t2[1] & 1) ? 7 : 1, nz = (r.t2[2] & 1) ? 7 : 1;
    const int x0 = (r.t2[0] & 1) ? 0 : r.t2[0] / 2, y0 = (r.t2[1] & 1) ? 0 : r.t2[1] / 2,
              z0 = (r.t2[2] & 1) ? 0 : r.t2[2] / 2;
    for (int c = 0; c < nz; ++c)
      for (int b = 0; b < ny; ++b)
        for (int a = 0; a < nx; ++a) {
          const int n = (x0 + a) + 7 * (y0 + b) + 49 * (z0 + c);
          const int32_t ds = depth_of[size_t(r.src_local) * NPT + n];
          if (o2n_local[size_t(r.src_local) * NPT + n] < 0) {
            if (ds < 0) throw BuildError{-2, "hanging chain out of order"};
            d = std::max(d, ds + 1);
          }
        }
    r.depth = d;
    depth_of[size_t(r.e_local) * NPT + r.node] = d;
  }
  std::stable_sort(hang_rows.begin(), hang_rows.end(),
                   [](const HangRow& a, const HangRow& b) { return a.depth < b.depth; });
}

// Padding sources of owned octants (R15): finest touching leaf whose
// closed box contains the point, lowest index on ties; outside a non-periodic
// domain -> extrapolation.
void HostMesh::build_padding() {
  const int64_t no = n_owned_oct;
  pmap.assign(size_t(no) * PMAP_PITCH, PM_EXTRAP);
  nbr.assign(size_t(no) * NBR_MAX, NbrEntry{0, {0, 0, 0}, 0, 0});
  n_nbr.assign(no, 0);
  pad_src_global.assign(size_t(no) * NPATCH, -1);
  pad_kind.assign(size_t(no) * NPATCH, 4);
  int bad = 0;
#pragma omp parallel for schedule(dynamic, 64) reduction(+ : bad)
  for (int64_t lb = 0; lb < no; ++lb) {
    const int64_t b = oct_begin + lb;
    const Oct& q = oct[b];
    const int64_t s = side(int32_t(b));
    uint8_t* pm = &pmap[size_t(lb) * PMAP_PITCH];
    int32_t* psrc = &pad_src_global[size_t(lb) * NPATCH];
    uint8_t* pk = &pad_kind[size_t(lb) * NPATCH];
    // outside flags per axis and patch index
    bool outside[3][P13];
    for (int k = 0; k < 3; ++k)
      for (int i = 0; i < P13; ++i) {
        const int64_t X = 6 * q.a[k] + (i - KPAD) * s;
        outside[k][i] = !periodic && (X < 0 || X > L);
      }
    std::vector<int> best_l(NPATCH, -1);
    std::vector<int32_t> best_c(NPATCH, INT32_MAX);
    std::vector<int8_t> best_j(NPATCH, -1);
    for (int p = 0; p < NPATCH; ++p) {
      const int i = p % 13, j = (p / 13) % 13, k = p / 169;
      const bool interior = i >= 3 && i <= 9 && j >= 3 && j <= 9 && k >= 3 && k <= 9;
      if (interior) {
        pm[p] = PM_SELF;
        psrc[p] = int32_t(b);
        pk[p] = 0;
      }
    }
    const std::vector<Touch>& tl = touch[b];
    for (size_t jt = 0; jt < tl.size(); ++jt) {
      const Touch& t = tl[jt];
      const Oct& c = oct[t.leaf];
      const int64_t sc = side(t.leaf);
      int lo_i[3], hi_i[3];
      for (int k = 0; k < 3; ++k) {
        const int64_t lo = 6 * c.a[k] + t.sh[k] - 6 * q.a[k];
        const int64_t hi = lo + 6 * sc;
        // patch index i is inside iff lo <= (i-3) s <= hi
        int64_t a0 = lo >= 0 ? (lo + s - 1) / s : -((-lo) / s);
        int64_t a1 = hi >= 0 ? hi / s : -((-hi + s - 1) / s);
        lo_i[k] = int(std::max<int64_t>(a0 + KPAD, 0));
        hi_i[k] = int(std::min<int64_t>(a1 + KPAD, P13 - 1));
      }
      for (int kk = lo_i[2]; kk <= hi_i[2]; ++kk)
        for (int jj = lo_i[1]; jj <= hi_i[1]; ++jj)
          for (int ii = lo_i[0]; ii <= hi_i[0]; ++ii) {
            const int p = ii + 13 * jj + 169 * kk;
            if (pm[p] == PM_SELF) continue;
            if (outside[0][ii] || outside[1][jj] || outside[2][kk]) continue;
            if (c.l > best_l[p] || (c.l == best_l[p] && t.leaf < best_c[p])) {
              best_l[p] = c.l;
              best_c[p] = t.leaf;
              best_j[p] = int8_t(jt);
            }
          }
    }
    // compact neighbour table of the entries actually used
    int8_t remap[NBR_MAX];
    for (int jt = 0; jt < NBR_MAX; ++jt) remap[jt] = -1;
    int nn = 0;
    for (int p = 0; p < NPATCH; ++p) {
      if (pm[p] == PM_SELF) continue;
      const int i = p % 13, j = (p / 13) % 13, k = p / 169;
      if (outside[0][i] || outside[1][j] || outside[2][k]) {
        pm[p] = PM_EXTRAP;
        psrc[p] = -1;
        pk[p] = 4;
        continue;
      }
      const int jt = best_j[p];
      if (jt < 0) {
        ++bad;
        continue;
      }
      if (remap[jt] < 0) remap[jt] = int8_t(nn++);
      pm[p] = uint8_t(remap[jt]);
      const Touch& t = tl[jt];
      const int cl = oct[t.leaf].l;
      uint8_t kd = cl == q.l ? 1 : (cl > q.l ? 2 : 3);
      if (t.sh[0] || t.sh[1] || t.sh[2]) kd |= 8;
      psrc[p] = t.leaf;
      pk[p] = kd;
    }
    n_nbr[lb] = nn;
    for (size_t jt = 0; jt < tl.size(); ++jt) {
      if (remap[jt] < 0) continue;
      const Touch& t = tl[jt];
      const int64_t sc = side(t.leaf);
      NbrEntry ne;
      ne.src = g2l_oct[t.leaf];
      if (ne.src < 0) ++bad;
      ne.r = uint8_t(2 * s / sc);
      for (int k = 0; k < 3; ++k) {
        const int64_t num = 2 * (6 * q.a[k] - KPAD * s - t.sh[k] - 6 * oct[t.leaf].a[k]);
        if (num % sc) ++bad;
        ne.o[k] = int16_t(num / sc);
      }
      ne.pad = 0;
      ne.pad2[0] = ne.pad2[1] = 0;
      for (int k = 0; k < 3; ++k) {
        ne.lo[k] = 12;
        ne.hi[k] = 0;
      }
      nbr[size_t(lb) * NBR_MAX + remap[jt]] = ne;
    }
    for (int p = 0; p < NPATCH; ++p) {
      const int jn = pm[p];
      if (jn >= nn) continue;
      NbrEntry& ne = nbr[size_t(lb) * NBR_MAX + jn];
      const int idx[3] = {p % 13, (p / 13) % 13, p / 169};
      for (int k = 0; k < 3; ++k) {
        ne.lo[k] = uint8_t(std::min<int>(ne.lo[k], idx[k]));
        ne.hi[k] = uint8_t(std::max<int>(ne.hi[k], idx[k]));
      }
    }
    // a coarser source (twice the octant's size) spans at most 10 patch indices per
    // axis; the device sweep buffers rely on it
    for (int jn = 0; jn < nn; ++jn) {
      const NbrEntry& ne = nbr[size_t(lb) * NBR_MAX + jn];
      if (ne.r == 1) {
        int thin = 13;
        for (int k = 0; k < 3; ++k) {
          if (ne.hi[k] - ne.lo[k] + 1 > 10) ++bad;
          thin = std::min(thin, ne.hi[k] - ne.lo[k] + 1);
        }
        // it lies beyond one face: 3 padding layers + the face plane itself
        if (thin > 4) ++bad;
      }
    }
  }
  if (bad) throw BuildError{-2, "padding map construction failed"};
}

void HostMesh::build(const double xmin_[3], double width_, int D_, bool periodic_,
                     const std::vector<Oct>& leaves, int rank_, int nranks_) {
  for (int k = 0; k < 3; ++k) xmin[k] = xmin_[k];
  width = width_;
  D = D_;
  periodic = periodic_;
  L = 6 * (int64_t(1) << D);
  oct = leaves;
  rank = rank_;
  nranks = nranks_;
  if (D < 1 || D > 20) throw BuildError{-1, "max_depth must be in 1..20"};
  if (nranks < 1 || rank < 0 || rank >= nranks) throw BuildError{-1, "bad rank/nranks"};
  if (int64_t(leaves.size()) < nranks) throw BuildError{-1, "fewer octants than ranks"};
  validate();
  build_touch();
  classify_nodes();
  partition();
  build_padding();
}

}  // namespace dgr
