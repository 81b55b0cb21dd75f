// Host-side octree and map construction for libdgr (C++17, OpenMP).
//
// Builds, for a balanced Morton-ordered linear octree, the maps the
// device path needs (P:L177-184 O2O/O2N, P:L241 O2P):
//   * touching-leaf lists (face/edge/corner neighbours, with periodic shifts)
//   * node classification: DOF / hanging, first-sight DOF numbering, hanging
//     sources with their half-grid coordinates, zip owners
//   * per-octant padding-source tables (the gather form of O2P)
//   * a Morton-contiguous partition with ghost octants / ghost DOFs.
// Definitions and tie-breaks: DESIGN.md §Maps (readings R14-R19).
// This is an independent implementation of the same definitions the oracle
// follows; the two are compared bit-for-bit on the exported maps.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace dgr {

constexpr int R = 7;         // points per octant edge
constexpr int KPAD = 3;      // padding width
constexpr int P13 = 13;      // patch edge
constexpr int NPT = 343;     // 7^3
constexpr int NPATCH = 2197; // 13^3
constexpr int NBR_MAX = 64;  // max touching (leaf, shift) entries per octant
constexpr uint8_t PM_SELF = 254, PM_EXTRAP = 255;
constexpr int PMAP_PITCH = 2208;  // bytes per octant in the device padding map (16-B rows)

struct Oct {
  int64_t a[3];
  int l;
};

struct Touch {
  int32_t leaf;
  int64_t sh[3];  // periodic shift of the leaf's box, node-lattice units
};

struct HangRef {      // hanging node (e, n): value = I_src at half-grid t2
  int32_t src;
  uint8_t t2[3];
};

// Device-side neighbour entry: t2_d(i) = o[d] + r * i for patch index i.
struct NbrEntry {
  int32_t src;   // local octant index
  int16_t o[3];
  uint8_t r;     // 1 (source coarser), 2 (same level), 4 (finer)
  uint8_t pad;
  uint8_t lo[3], hi[3];  // bounding box (patch indices) of the points it sources
  uint8_t pad2[2];
};
static_assert(sizeof(NbrEntry) == 20, "NbrEntry layout");

struct BuildError {
  int code;
  std::string msg;
};

class HostMesh {
 public:
  // geometry
  double xmin[3] = {0, 0, 0};
  double width = 1.0;
  int D = 18;
  bool periodic = false;
  int64_t L = 0;  // node-lattice extent 6 * 2^D

  std::vector<Oct> oct;          // global leaves, Morton order
  std::vector<uint64_t> key;     // Morton keys of anchors
  std::vector<std::vector<Touch>> touch;

  // global node maps, [N * 343]
  std::vector<int32_t> o2n;      // global DOF id or -1
  std::vector<HangRef> hang;     // valid where o2n == -1
  int64_t n_dof = 0;
  std::vector<int32_t> zip_leaf, zip_node;  // per global DOF

  int level_min = 0, level_max = 0;

  // partition
  int rank = 0, nranks = 1;
  int64_t oct_begin = 0, oct_end = 0;          // owned global range
  std::vector<int32_t> local_oct;              // local -> global octant
  std::vector<int32_t> g2l_oct;                // global -> local (-1)
  int64_t n_owned_oct = 0, n_ghost_oct = 0;
  std::vector<int64_t> dof_gid;                // local DOF -> global id
  int64_t n_owned_dof = 0, n_ghost_dof = 0;
  std::vector<int32_t> dof_owner_rank;         // per global DOF
  std::vector<int64_t> recv_counts, send_counts;  // per peer
  std::vector<int32_t> send_list;              // local DOF ids, peer-major

  // per local octant (owned + ghost) maps in local numbering
  std::vector<int32_t> o2n_local;              // [n_local * 343] local DOF or -1
  // per owned octant padding tables
  std::vector<uint8_t> pmap;                   // [n_owned * PMAP_PITCH]
  std::vector<NbrEntry> nbr;                   // [n_owned * NBR_MAX]
  std::vector<int32_t> n_nbr;                  // [n_owned]
  std::vector<int32_t> pad_src_global;         // [n_owned * 2197] export
  std::vector<uint8_t> pad_kind;               // [n_owned * 2197] export
  // hanging rows over local octants, sorted by (level, local octant, node)
  struct HangRow {
    int32_t e_local, node, src_local;
    uint8_t t2[3];
    int level, depth;
    int32_t e_global, src_global;
  };
  std::vector<HangRow> hang_rows;
  // zip: owned DOF -> local octant * 343 + node
  std::vector<int32_t> zip_local;

  // Build from a validated octant list. Throws BuildError.
  void build(const double xmin_[3], double width_, int D_, bool periodic_,
             const std::vector<Oct>& leaves, int rank_, int nranks_);

  int32_t locate(int64_t cx, int64_t cy, int64_t cz) const;  // leaf containing cell; -1 outside
  int64_t side(int32_t e) const { return int64_t(1) << (D - oct[e].l); }

 private:
  void validate();
  void build_touch();
  void classify_nodes();
  void partition();
  void build_padding();
};

uint64_t morton(int64_t x, int64_t y, int64_t z, int D);

// Refinement rule + minimal 2:1 vertex balance + Morton sort.
struct PunctureDesc {
  double x, y, z, m;
  int level;
};
std::vector<Oct> build_octree(const double xmin[3], double width, int D, bool periodic,
                              int level_min, const std::vector<PunctureDesc>& punct, double rho);

// Regrid (readings R30-R32): new leaves from the per-leaf wavelet
// indicator w (global Morton order) — split above eps_refine, merge complete
// sibling families below eps_coarsen — then the minimal 2:1 balance closure.
std::vector<Oct> regrid_leaves(const std::vector<Oct>& leaves, const double* w, double eps_refine,
                              double eps_coarsen, int level_min, int level_max, int D,
                              bool periodic);

}  // namespace dgr
