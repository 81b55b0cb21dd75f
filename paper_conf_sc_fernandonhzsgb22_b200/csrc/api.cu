// C ABI of libdgr (include/dgr.h): mesh lifetime, map export, and the
// device entry points (unzip, rhs, rk4 stage/step, constraints).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <array>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <new>
#include <string>
#include <vector>

#include "../../include/dgr.h"
#include "device.cuh"
#include "host_mesh.hpp"

namespace dgr {
void upload_tables(const double* w13, const double* wext);
}

using namespace dgr;

// --------------------------------------------------------------- errors
static thread_local std::string g_err;

static dgr_status fail(dgr_status s, const std::string& msg) {
  g_err = msg;
  return s;
}

#define CUDA_TRY(x)                                                                   \
  do {                                                                                \
    cudaError_t _e = (x);                                                             \
    if (_e != cudaSuccess)                                                            \
      return fail(_e == cudaErrorMemoryAllocation ? DGR_ERR_OOM : DGR_ERR_CUDA,       \
                  std::string(#x) + ": " + cudaGetErrorString(_e));                   \
  } while (0)

// ---------------------------------------------------------------- NCCL (dlopen)
namespace {
typedef int ncclResult_t_;
struct NcclApi {
  void* h = nullptr;
  ncclResult_t_ (*CommInitRank)(void**, int, const void* /*by value 128B*/, int) = nullptr;
  ncclResult_t_ (*CommDestroy)(void*) = nullptr;
  ncclResult_t_ (*Send)(const void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  ncclResult_t_ (*Recv)(void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  ncclResult_t_ (*GroupStart)() = nullptr;
  ncclResult_t_ (*GroupEnd)() = nullptr;
  ncclResult_t_ (*AllReduce)(const void*, void*, size_t, int, int, void*, cudaStream_t) = nullptr;
};
struct UniqueId {
  char internal[128];
};
typedef int (*InitRankFn)(void**, int, UniqueId, int);
InitRankFn g_init_rank = nullptr;
NcclApi g_nccl;
bool load_nccl() {
  if (g_nccl.h) return true;
  const char* names[] = {"libnccl.so.2", "libnccl.so"};
  for (const char* n : names) {
    g_nccl.h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
    if (g_nccl.h) break;
  }
  if (!g_nccl.h) return false;
  g_init_rank = (InitRankFn)dlsym(g_nccl.h, "ncclCommInitRank");
  g_nccl.CommDestroy = (ncclResult_t_(*)(void*))dlsym(g_nccl.h, "ncclCommDestroy");
  g_nccl.Send = (ncclResult_t_(*)(const void*, size_t, int, int, void*, cudaStream_t))dlsym(
      g_nccl.h, "ncclSend");
  g_nccl.Recv =
      (ncclResult_t_(*)(void*, size_t, int, int, void*, cudaStream_t))dlsym(g_nccl.h, "ncclRecv");
  g_nccl.GroupStart = (ncclResult_t_(*)())dlsym(g_nccl.h, "ncclGroupStart");
  g_nccl.GroupEnd = (ncclResult_t_(*)())dlsym(g_nccl.h, "ncclGroupEnd");
  g_nccl.AllReduce = (ncclResult_t_(*)(const void*, void*, size_t, int, int, void*,
                                       cudaStream_t))dlsym(g_nccl.h, "ncclAllReduce");
  return g_init_rank && g_nccl.Send && g_nccl.Recv && g_nccl.GroupStart && g_nccl.GroupEnd &&
         g_nccl.AllReduce && g_nccl.CommDestroy;
}
constexpr int NCCL_FLOAT64 = 8, NCCL_SUM = 0, NCCL_MAX = 2;
}  // namespace

// ----------------------------------------------------------------- mesh
struct dgr_group_s;
struct dgr_mesh_s {
  HostMesh host;
  bool device = false;
  int dev_id = -1;
  DevMesh dm{};
  double xmin[3];
  // device allocations
  std::vector<void*> allocs;
  int4* d_oct = nullptr;
  int32_t* d_o2n = nullptr;
  uint8_t* d_pmap = nullptr;
  NbrEntry* d_nbr = nullptr;
  int32_t* d_zip = nullptr;
  int32_t* d_own = nullptr;     // [n_owned*343] zip-owned DOF of each point or -1
  int64_t* d_dof_node = nullptr;
  double* d_aux = nullptr;      // [24][aux_stride] interpolation slots
  int32_t* d_o2s = nullptr;     // [n_local][343] element node -> u / slot index
  int32_t* d_gmap = nullptr;    // [n_owned][GM_PITCH] patch point -> u / slot index
  int32_t* d_gmap_s = nullptr;  // [n_owned][GM_PITCH] the same entries sorted by source
  int16_t* d_gdst = nullptr;    // [n_owned][GM_PITCH] patch point of each sorted entry
  // k_interp launch ranges, one per dependency depth, per phase: phase 0 =
  // slot elements whose values depend on owned DOFs only, phase 1 = the rest
  // (they wait for the ghost exchange; empty on one rank)
  std::vector<int64_t> iel_depth_off[2];
  // RHS octant order: olist[0, n_interior) need no ghost value (they run while
  // the ghost exchange is in flight), olist[n_interior, n_owned) the rest
  int32_t* d_olist = nullptr;
  int64_t n_interior = 0;
  cudaStream_t xstream = nullptr;   // ghost exchange stream (N > 1)
  int xsm = 8;                      // SMs k_rhs leaves to NCCL while overlapping
  int phases = 0;                   // DGR_OPT_PHASES
  bool prepass = true;              // DGR_OPT_PREPASS: gt_ij stages in k_gt_pre
  bool zip_store = true;            // DGR_OPT_ZIP_STORE: k_rhs stores in DOF order
  double* d_rhs_dof = nullptr;      // [24][dof_stride] RHS in DOF order (RK4 stages)
  double* d_pre = nullptr;          // [30][n_owned][352] metric pre-pass results (by thread)
  cudaEvent_t ev_ready = nullptr, ev_xdone = nullptr;
  int4* d_iel = nullptr;        // interpolation work per element with slots
  int4* d_igrp = nullptr;       // ... per face group of its slots
  uint16_t* d_ipt = nullptr;    // half-grid point of each interpolation slot
  int64_t n_interp = 0;
  double* d_patch = nullptr;    // [24][n_owned][PATCH_PITCH] (allocated on first dgr_unzip)
  double* d_rhs_oct = nullptr;  // [24][n_owned][343]
  double* d_us = nullptr;       // RK4 stage state [24][dof_stride]
  double* d_acc = nullptr;      // RK4 accumulator
  double* d_cnorm = nullptr;    // constraint norm partials
  // Psi_4 extraction (allocated on first use): inputs [234][n], positions [3][n],
  // Psi_4 at the octant nodes [2][n], n = n_owned * 343
  double* d_psi_in = nullptr;
  double* d_psi_xyz = nullptr;
  double* d_psi = nullptr;
  // dgr_rk4_step_host: three device state slots, copy streams and events
  // (allocated on first use)
  double* d_hbuf[3] = {nullptr, nullptr, nullptr};
  cudaStream_t h2d = nullptr, d2h = nullptr;
  cudaEvent_t ev_in[3] = {}, ev_done[3] = {}, ev_out[3] = {}, ev_host0 = nullptr;
  // multi-rank: peer-major send / receive buffers (one [NF][n_p] block per
  // peer p), per-peer prefix offsets, NCCL communicator or in-process group
  void* comm = nullptr;
  dgr_group_s* group = nullptr;     // linked in-process ranks (dgr_group_create)
  int32_t* d_send = nullptr;
  double* d_sendbuf = nullptr;
  double* d_recvbuf = nullptr;
  PeerOffsets po_send{}, po_recv{};
  int64_t launches = 0;
  bool fused = true;            // DGR_OPT_FUSED_UNZIP (C3: 40.4 ms/step fused, 41.2 two-pass)
  // DGR_OPT_GRAPH: dgr_rk4_step replays a CUDA graph of its 4 stages (captured
  // on a library stream at the second call with the same arguments)
  bool use_graph = true;
  // DGR_OPT_FUSE_RK4: dgr_rk4_step / dgr_rk4_step_host apply the RK4 stage
  // update in k_rhs's zip-by-store epilogue (no k_rk4), the stage states
  // alternating between d_us and d_us2 (a stage never writes what it gathers)
  bool fuse_rk4 = true;
  double* d_us2 = nullptr;
  cudaStream_t gstream = nullptr;
  cudaGraphExec_t gexec = nullptr;
  int64_t glaunches = 0;
  struct GraphKey { const double* u; double dt; dgr_params prm; bool has_prm; } gkey{};
  int gseen = 0;                // calls with the current key (0: none)
  void drop_graph() {
    if (gexec) cudaGraphExecDestroy(gexec);
    gexec = nullptr;
    gseen = 0;
  }
  // profiling
  bool prof = false;
  struct Pend { int cls; cudaEvent_t a, b; };
  std::vector<Pend> pend;
  std::vector<cudaEvent_t> pool;
  double prof_ms[DGR_PROF_CLASSES] = {0};
  int64_t prof_n[DGR_PROF_CLASSES] = {0};
  cudaEvent_t ev() {
    if (!pool.empty()) { cudaEvent_t e = pool.back(); pool.pop_back(); return e; }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
  }

  template <class T>
  cudaError_t alloc(T** p, size_t n) {
    void* q = nullptr;
    cudaError_t e = cudaMalloc(&q, std::max<size_t>(n, 1) * sizeof(T));
    if (e == cudaSuccess) {
      allocs.push_back(q);
      *p = static_cast<T*>(q);
    }
    return e;
  }
  ~dgr_mesh_s() {
    for (auto& p : pend) { cudaEventDestroy(p.a); cudaEventDestroy(p.b); }
    for (auto e : pool) cudaEventDestroy(e);
    for (void* q : allocs) cudaFree(q);
    if (comm && g_nccl.CommDestroy) g_nccl.CommDestroy(comm);
    if (ev_ready) cudaEventDestroy(ev_ready);
    if (ev_xdone) cudaEventDestroy(ev_xdone);
    if (xstream) cudaStreamDestroy(xstream);
    for (int b = 0; b < 3; ++b) {
      if (ev_in[b]) cudaEventDestroy(ev_in[b]);
      if (ev_done[b]) cudaEventDestroy(ev_done[b]);
      if (ev_out[b]) cudaEventDestroy(ev_out[b]);
    }
    if (ev_host0) cudaEventDestroy(ev_host0);
    if (gexec) cudaGraphExecDestroy(gexec);
    if (gstream) cudaStreamDestroy(gstream);
    if (h2d) cudaStreamDestroy(h2d);
    if (d2h) cudaStreamDestroy(d2h);
  }
};

// Lagrange rows computed exactly: l_m(t2/2) = prod_{q!=m} (t2 - 2q) / (2 (m - q)).
static void lagrange_tables(double* w13, double* wext) {
  for (int t2 = 0; t2 < 13; ++t2)
    for (int m = 0; m < 7; ++m) {
      long long num = 1, den = 1;
      for (int q = 0; q < 7; ++q)
        if (q != m) {
          num *= (t2 - 2 * q);
          den *= 2 * (m - q);
        }
      w13[t2 * 7 + m] = double(num) / double(den);
    }
  for (int t = 0; t < 3; ++t) {
    const int tt = -(t + 1);
    for (int m = 0; m < 7; ++m) {
      long long num = 1, den = 1;
      for (int q = 0; q < 7; ++q)
        if (q != m) {
          num *= (tt - q);
          den *= (m - q);
        }
      wext[t * 7 + m] = double(num) / double(den);
    }
  }
}

extern "C" {

const char* dgr_status_string(dgr_status s) {
  switch (s) {
    case DGR_OK: return "ok";
    case DGR_ERR_ARG: return "invalid argument";
    case DGR_ERR_TREE: return "invalid octree";
    case DGR_ERR_CUDA: return "CUDA error";
    case DGR_ERR_NCCL: return "NCCL error";
    case DGR_ERR_OOM: return "out of memory";
    case DGR_ERR_STATE: return "invalid state";
  }
  return "unknown";
}

const char* dgr_last_error(void) { return g_err.c_str(); }
const char* dgr_version(void) { return "dgr-b200 0.1 (sm_100a)"; }

dgr_status dgr_octree_build(const dgr_refine_desc* desc, dgr_octant* out, int64_t* n_inout) {
  if (!desc || !n_inout) return fail(DGR_ERR_ARG, "null argument");
  if (desc->max_depth < 1 || desc->max_depth > 20 || desc->width <= 0 || desc->n_punct < 0 ||
      (desc->n_punct > 0 && !desc->punct) || desc->level_min < 0 ||
      desc->level_min > desc->max_depth)
    return fail(DGR_ERR_ARG, "bad refine descriptor");
  try {
    std::vector<PunctureDesc> p;
    for (int i = 0; i < desc->n_punct; ++i) {
      const dgr_puncture& q = desc->punct[i];
      if (q.level < 0 || q.level > desc->max_depth) return fail(DGR_ERR_ARG, "bad puncture level");
      p.push_back({q.x, q.y, q.z, q.m, q.level});
    }
    std::vector<Oct> o = build_octree(desc->xmin, desc->width, desc->max_depth,
                                      desc->periodic != 0, desc->level_min, p, desc->rho);
    if (!out) {
      *n_inout = int64_t(o.size());
      return DGR_OK;
    }
    if (*n_inout < int64_t(o.size())) return fail(DGR_ERR_ARG, "output buffer too small");
    for (size_t i = 0; i < o.size(); ++i)
      out[i] = {uint32_t(o[i].a[0]), uint32_t(o[i].a[1]), uint32_t(o[i].a[2]), uint32_t(o[i].l)};
    *n_inout = int64_t(o.size());
    return DGR_OK;
  } catch (const std::bad_alloc&) {
    return fail(DGR_ERR_OOM, "host allocation failed");
  }
}

static dgr_status upload(dgr_mesh m, cudaStream_t st) {
  HostMesh& h = m->host;
  const int64_t nl = int64_t(h.local_oct.size());
  const int64_t no = h.n_owned_oct;
  CUDA_TRY(cudaGetDevice(&m->dev_id));
  // octant info
  std::vector<int4> oi(nl);
  for (int64_t l = 0; l < nl; ++l) {
    const Oct& o = h.oct[h.local_oct[l]];
    oi[l] = make_int4(int(o.a[0]), int(o.a[1]), int(o.a[2]), o.l);
  }
  CUDA_TRY(m->alloc(&m->d_oct, nl));
  CUDA_TRY(cudaMemcpy(m->d_oct, oi.data(), nl * sizeof(int4), cudaMemcpyHostToDevice));
  CUDA_TRY(m->alloc(&m->d_o2n, h.o2n_local.size()));
  CUDA_TRY(cudaMemcpy(m->d_o2n, h.o2n_local.data(), h.o2n_local.size() * 4, cudaMemcpyHostToDevice));
  CUDA_TRY(m->alloc(&m->d_pmap, h.pmap.size()));
  CUDA_TRY(cudaMemcpy(m->d_pmap, h.pmap.data(), h.pmap.size(), cudaMemcpyHostToDevice));
  CUDA_TRY(m->alloc(&m->d_nbr, h.nbr.size()));
  CUDA_TRY(cudaMemcpy(m->d_nbr, h.nbr.data(), h.nbr.size() * sizeof(NbrEntry),
                      cudaMemcpyHostToDevice));
  {
    // inverse zip map for the fused RHS epilogue: point -> owned DOF it is the zip owner of
    std::vector<int32_t> own(size_t(no) * NPT, -1);
    for (size_t l = 0; l < h.zip_local.size(); ++l) own[h.zip_local[l]] = int32_t(l);
    CUDA_TRY(m->alloc(&m->d_own, own.size()));
    CUDA_TRY(cudaMemcpy(m->d_own, own.data(), own.size() * 4, cudaMemcpyHostToDevice));
  }
  CUDA_TRY(m->alloc(&m->d_zip, h.zip_local.size()));
  CUDA_TRY(cudaMemcpy(m->d_zip, h.zip_local.data(), h.zip_local.size() * 4, cudaMemcpyHostToDevice));
  // DOF lattice coordinates
  const int64_t nd = h.n_owned_dof + h.n_ghost_dof;
  const int64_t stride = ((nd + 31) / 32) * 32;
  std::vector<int64_t> node(3 * stride, 0);
  for (int64_t d = 0; d < nd; ++d) {
    const int64_t g = h.dof_gid[d];
    const int32_t e = h.zip_leaf[g], n = h.zip_node[g];
    const Oct& o = h.oct[e];
    const int64_t s = h.side(e);
    node[3 * d + 0] = 6 * o.a[0] + (n % 7) * s;
    node[3 * d + 1] = 6 * o.a[1] + ((n / 7) % 7) * s;
    node[3 * d + 2] = 6 * o.a[2] + (n / 49) * s;
  }
  CUDA_TRY(m->alloc(&m->d_dof_node, node.size()));
  CUDA_TRY(cudaMemcpy(m->d_dof_node, node.data(), node.size() * 8, cudaMemcpyHostToDevice));
  // Gather maps.  Every value a patch needs is either a DOF of
  // the state u (index < dof_stride) or an interpolation SLOT of the auxiliary
  // array (index dof_stride + slot): one slot per distinct (coarse element c,
  // half-grid point t2 of c) that is needed, either by a hanging node of a finer
  // element (Alg. 2 lines 4-5) or by a padding point sourced by a
  // coarser neighbour.  o2s[e][n] maps element nodes to that index
  // space; gmap[e][p] maps patch points (copy / injection through o2s of the
  // source element, interpolation to its slot, -1 = extrapolated).  Slots are
  // numbered by dependency depth (a slot of c whose 343 nodes are all DOFs has
  // depth 0, else 1 + the deepest slot among c's nodes; reading R14), then
  // element, then t2 — k_interp fills one depth per launch.
  const int64_t ds = ((h.n_owned_dof + h.n_ghost_dof + 31) / 32) * 32;
  int64_t aux_stride = 0;
  {
    std::vector<int32_t> cid(size_t(nl), -1);        // element -> need table
    std::vector<std::vector<int32_t>> need;          // [t2x + 13 t2y + 169 t2z] -> -1 / -2 / slot
    std::vector<int32_t> celem;
    auto mark = [&](int32_t c, int q) {
      if (cid[c] < 0) {
        cid[c] = int32_t(need.size());
        need.emplace_back(NPATCH, -1);
        celem.push_back(c);
      }
      need[cid[c]][q] = -2;
    };
    // hanging nodes
    std::vector<int32_t> hsrc(size_t(nl) * NPT, -1);
    std::vector<int16_t> hq(size_t(nl) * NPT, -1);
    for (const auto& r : h.hang_rows) {
      if (r.t2[0] > 12 || r.t2[1] > 12 || r.t2[2] > 12)
        return fail(DGR_ERR_TREE, "hanging node outside its source element");
      const int q = r.t2[0] + 13 * r.t2[1] + 169 * r.t2[2];
      hsrc[size_t(r.e_local) * NPT + r.node] = r.src_local;
      hq[size_t(r.e_local) * NPT + r.node] = int16_t(q);
      mark(r.src_local, q);
    }
    // padding points sourced by a coarser neighbour
    for (int64_t e = 0; e < no; ++e) {
      const uint8_t* pm = h.pmap.data() + size_t(e) * PMAP_PITCH;
      const NbrEntry* nb = h.nbr.data() + size_t(e) * NBR_MAX;
      for (int p = 0; p < NPATCH; ++p) {
        const int j = pm[p];
        if (j == PM_SELF || j == PM_EXTRAP || nb[j].r != 1) continue;
        const NbrEntry& t = nb[j];
        const int tx = t.o[0] + p % 13, ty = t.o[1] + (p / 13) % 13, tz = t.o[2] + p / 169;
        if (tx < 0 || tx > 12 || ty < 0 || ty > 12 || tz < 0 || tz > 12)
          return fail(DGR_ERR_TREE, "interpolation point outside its source element");
        mark(t.src, tx + 13 * ty + 169 * tz);
      }
    }
    // dependency depth per slot element, coarse to fine (a hanging node's source is coarser)
    std::vector<int32_t> order(celem.size());
    for (size_t i = 0; i < order.size(); ++i) order[i] = int32_t(i);
    auto lev = [&](int32_t c) { return h.oct[h.local_oct[c]].l; };
    std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
      return lev(celem[a]) != lev(celem[b]) ? lev(celem[a]) < lev(celem[b]) : celem[a] < celem[b];
    });
    std::vector<int32_t> edepth(size_t(nl), -1);   // depth of the slots of element c
    auto node_depth = [&](int32_t e, int n) -> int32_t {   // -1: a DOF
      const int32_t src = hsrc[size_t(e) * NPT + n];
      return src < 0 ? -1 : edepth[src];
    };
    for (int32_t ci : order) {
      const int32_t c = celem[ci];
      int32_t d = 0;
      for (int n = 0; n < NPT; ++n) {
        const int32_t nd = node_depth(c, n);
        if (nd == -1) continue;
        if (edepth[hsrc[size_t(c) * NPT + n]] < 0)
          return fail(DGR_ERR_TREE, "hanging source not coarser than its element");
        d = std::max(d, nd + 1);
      }
      edepth[c] = d;
    }
    // remote dependency: a slot element needs a ghost value if one of its
    // nodes is a ghost DOF or a slot of such an element (coarse to fine)
    std::vector<uint8_t> erdep(size_t(nl), 0);
    for (int32_t ci : order) {
      const int32_t c = celem[ci];
      uint8_t r = 0;
      for (int n = 0; n < NPT && !r; ++n) {
        const size_t k = size_t(c) * NPT + n;
        const int32_t d = h.o2n_local[k];
        r = d >= 0 ? uint8_t(d >= h.n_owned_dof) : erdep[hsrc[k]];
      }
      erdep[c] = r;
    }
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
      const int32_t pa = erdep[celem[a]], pb = erdep[celem[b]];
      if (pa != pb) return pa < pb;
      const int32_t da = edepth[celem[a]], db = edepth[celem[b]];
      return da != db ? da < db : celem[a] < celem[b];
    });
    std::vector<int4> iel, igrp;
    std::vector<uint16_t> ipt;
    m->iel_depth_off[0].clear();
    m->iel_depth_off[1].clear();
    std::vector<uint8_t> slot_rdep;
    int64_t slot = 0;
    int prev_depth = -1, prev_phase = 0;
    for (int32_t ci : order) {
      const int32_t c = celem[ci];
      if (erdep[c] != prev_phase) {   // phase 0 -> 1
        m->iel_depth_off[0].push_back(int64_t(iel.size()));
        prev_phase = erdep[c];
        prev_depth = -1;
      }
      if (edepth[c] != prev_depth) {
        m->iel_depth_off[prev_phase].push_back(int64_t(iel.size()));
        prev_depth = edepth[c];
      }
      // one work entry per (element, face group): a slot belongs to the first
      // face (x-low, x-high, y-low, ...) it lies within 3 half-grid points of
      // (every slot does: hanging nodes lie on faces, padding reaches 1.5
      // coarse cells in), and its group sweeps that face's normal axis first
      // over a bounding box <= 4 points thick.  The sweep order is thus a
      // function of (element, point) alone, so a slot has the same value on
      // every partition (multi-rank bit identity).
      const int32_t g_first = int32_t(igrp.size());
      for (int grp = 0; grp < 6; ++grp) {
        int lo[3] = {12, 12, 12}, hi[3] = {0, 0, 0};
        const int64_t first = slot;
        for (int q = 0; q < NPATCH; ++q) {
          if (need[ci][q] != -2) continue;
          const int t[3] = {q % 13, (q / 13) % 13, q / 169};
          int g = -1;
          for (int a = 0; a < 3 && g < 0; ++a)
            g = t[a] <= 3 ? 2 * a : (t[a] >= 9 ? 2 * a + 1 : -1);
          if (g < 0) return fail(DGR_ERR_TREE, "interpolation point not near a face of its element");
          if (g != grp) continue;
          for (int k = 0; k < 3; ++k) {
            lo[k] = std::min(lo[k], t[k]);
            hi[k] = std::max(hi[k], t[k]);
          }
          need[ci][q] = int32_t(slot++);
          ipt.push_back(uint16_t(t[0] | (t[1] << 4) | (t[2] << 8)));
        }
        if (slot == first) continue;
        if (hi[grp / 2] - lo[grp / 2] + 1 > 4)   // k_interp's scratch bound (IP_N1)
          return fail(DGR_ERR_TREE, "interpolation face group thicker than 4 points");
        const int lohi = (lo[0] | (lo[1] << 4) | (lo[2] << 8)) |
                         ((hi[0] | (hi[1] << 4) | (hi[2] << 8)) << 12) | ((grp / 2) << 24);
        igrp.push_back(make_int4(int32_t(first), int32_t(slot - first), lohi, 0));
      }
      iel.push_back(make_int4(c, g_first, int32_t(igrp.size()) - g_first, 0));
      slot_rdep.resize(size_t(slot), erdep[c]);
    }
    m->iel_depth_off[prev_phase].push_back(int64_t(iel.size()));
    if (ds + slot >= (int64_t(1) << 31)) return fail(DGR_ERR_ARG, "mesh too large for int32 gather maps");
    // element nodes -> u / slot index
    std::vector<int32_t> o2s(size_t(nl) * NPT);
    for (int64_t e = 0; e < nl; ++e)
      for (int n = 0; n < NPT; ++n) {
        const size_t k = size_t(e) * NPT + n;
        const int32_t d = h.o2n_local[k];
        if (d >= 0) {
          o2s[k] = d;
        } else {
          if (hsrc[k] < 0) return fail(DGR_ERR_TREE, "hanging node without a source");
          o2s[k] = int32_t(ds + need[cid[hsrc[k]]][hq[k]]);
        }
      }
    // patch points -> u / slot index
    std::vector<int32_t> gm(size_t(no) * GM_PITCH, -1);
    for (int64_t e = 0; e < no; ++e) {
      const uint8_t* pm = h.pmap.data() + size_t(e) * PMAP_PITCH;
      const NbrEntry* nb = h.nbr.data() + size_t(e) * NBR_MAX;
      for (int p = 0; p < NPATCH; ++p) {
        const int j = pm[p];
        const int ix = p % 13, iy = (p / 13) % 13, iz = p / 169;
        int32_t v = -1;
        if (j == PM_SELF) {
          v = o2s[size_t(e) * NPT + (ix - 3) + 7 * (iy - 3) + 49 * (iz - 3)];
        } else if (j != PM_EXTRAP) {
          const NbrEntry& t = nb[j];
          if (t.r == 1) {
            const int q = (t.o[0] + ix) + 13 * (t.o[1] + iy) + 169 * (t.o[2] + iz);
            v = int32_t(ds + need[cid[t.src]][q]);
          } else {
            const int tx = (t.o[0] + t.r * ix) >> 1, ty = (t.o[1] + t.r * iy) >> 1,
                      tz = (t.o[2] + t.r * iz) >> 1;
            v = o2s[size_t(t.src) * NPT + tx + 7 * ty + 49 * tz];
          }
        }
        gm[size_t(e) * GM_PITCH + p] = v;
      }
    }
    // interior octants first (no gather source depends on a ghost value)
    {
      std::vector<int32_t> olist;
      olist.reserve(size_t(no));
      std::vector<int32_t> bnd;
      for (int64_t e = 0; e < no; ++e) {
        bool remote = false;
        const int32_t* row = gm.data() + size_t(e) * GM_PITCH;
        for (int p = 0; p < NPATCH && !remote; ++p) {
          const int32_t v = row[p];
          if (v < 0) continue;
          remote = v < ds ? v >= h.n_owned_dof : slot_rdep[size_t(v - ds)] != 0;
        }
        (remote ? bnd : olist).push_back(int32_t(e));
      }
      m->n_interior = int64_t(olist.size());
      olist.insert(olist.end(), bnd.begin(), bnd.end());
      CUDA_TRY(m->alloc(&m->d_olist, olist.size()));
      if (!olist.empty())
        CUDA_TRY(cudaMemcpy(m->d_olist, olist.data(), olist.size() * 4, cudaMemcpyHostToDevice));
    }
    m->n_interp = slot;
    aux_stride = std::max<int64_t>(32, ((slot + 31) / 32) * 32);
    CUDA_TRY(m->alloc(&m->d_o2s, o2s.size()));
    CUDA_TRY(cudaMemcpy(m->d_o2s, o2s.data(), o2s.size() * 4, cudaMemcpyHostToDevice));
    {
      // the fused kernels' gather order: each octant's entries sorted by source
      // index, so a warp's 32 copies read few distinct lines (fewer
      // shared-memory write wavefronts per cp.async); gdst keeps the patch point
      std::vector<int32_t> gs(gm.size(), -1);
      std::vector<int16_t> gd(gm.size(), 0);
      std::vector<int> idx(NPATCH);
      for (int64_t e = 0; e < no; ++e) {
        const int32_t* row = gm.data() + size_t(e) * GM_PITCH;
        // groups: cross points (at most one coordinate in the padding: all a
        // first-derivative stencil reads, G_CROSS of them), then the slabs
        // (two: the rest of what the D1 pass and mixed stencils read,
        // G_SLABS in total), then the 216 corners (read by nothing); sorted
        // by source inside each group
        auto grp = [](int p) {
          const int t[3] = {p % 13, (p / 13) % 13, p / 169};
          int out = 0;
          for (int a = 0; a < 3; ++a) out += (t[a] < 3 || t[a] > 9);
          return out <= 1 ? 0 : (out == 2 ? 1 : 2);
        };
        for (int p = 0; p < NPATCH; ++p) idx[p] = p;
        std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) {
          const int ga = grp(a), gb = grp(b);
          return ga != gb ? ga < gb : row[a] < row[b];
        });
        // (interleaving the entries by shared-memory bank pair to remove the
        // cp.async write conflicts measured slower — k_rhs 5.58 -> 5.97 ms:
        // the data-pipe wavefronts follow the number of global lines a warp's
        // 32 copies touch, which the source order minimises)
        for (int k = 0; k < NPATCH; ++k) {
          gs[size_t(e) * GM_PITCH + k] = row[idx[k]];
          gd[size_t(e) * GM_PITCH + k] = int16_t(idx[k]);
        }
      }
      CUDA_TRY(m->alloc(&m->d_gmap_s, gs.size()));
      CUDA_TRY(cudaMemcpy(m->d_gmap_s, gs.data(), gs.size() * 4, cudaMemcpyHostToDevice));
      CUDA_TRY(m->alloc(&m->d_gdst, gd.size()));
      CUDA_TRY(cudaMemcpy(m->d_gdst, gd.data(), gd.size() * 2, cudaMemcpyHostToDevice));
    }
    CUDA_TRY(m->alloc(&m->d_gmap, gm.size()));
    CUDA_TRY(cudaMemcpy(m->d_gmap, gm.data(), gm.size() * 4, cudaMemcpyHostToDevice));
    CUDA_TRY(m->alloc(&m->d_iel, iel.size()));
    if (!iel.empty())
      CUDA_TRY(cudaMemcpy(m->d_iel, iel.data(), iel.size() * sizeof(int4), cudaMemcpyHostToDevice));
    CUDA_TRY(m->alloc(&m->d_igrp, igrp.size()));
    if (!igrp.empty())
      CUDA_TRY(cudaMemcpy(m->d_igrp, igrp.data(), igrp.size() * sizeof(int4), cudaMemcpyHostToDevice));
    CUDA_TRY(m->alloc(&m->d_ipt, ipt.size()));
    if (!ipt.empty())
      CUDA_TRY(cudaMemcpy(m->d_ipt, ipt.data(), ipt.size() * 2, cudaMemcpyHostToDevice));
    m->dm.n_iel = int32_t(iel.size());
  }
  // workspace
  CUDA_TRY(m->alloc(&m->d_aux, size_t(NF) * aux_stride));
  CUDA_TRY(m->alloc(&m->d_rhs_oct, size_t(NF) * no * NPT));
  CUDA_TRY(m->alloc(&m->d_us, size_t(NF) * stride));
  CUDA_TRY(m->alloc(&m->d_acc, size_t(NF) * stride));
  CUDA_TRY(cudaMemset(m->d_aux, 0, size_t(NF) * aux_stride * 8));
  CUDA_TRY(cudaMemset(m->d_us, 0, size_t(NF) * stride * 8));
  CUDA_TRY(cudaMemset(m->d_acc, 0, size_t(NF) * stride * 8));
  double w13[91], wext[21];
  lagrange_tables(w13, wext);
  upload_tables(w13, wext);
  upload_rhs_tables(wext);
  upload_regrid_tables(w13);
  CUDA_TRY(cudaGetLastError());
  DevMesh& dm = m->dm;
  dm.n_owned = int32_t(no);
  dm.n_local = int32_t(nl);
  dm.dof_stride = stride;
  dm.n_owned_dof = int32_t(h.n_owned_dof);
  dm.D = h.D;
  dm.periodic = h.periodic ? 1 : 0;
  dm.width = h.width;
  for (int a = 0; a < 3; ++a) dm.xmin[a] = h.xmin[a];
  dm.oct = m->d_oct;
  dm.o2n = m->d_o2n;
  dm.pmap = m->d_pmap;
  dm.nbr = m->d_nbr;
  dm.zip = m->d_zip;
  dm.own = m->d_own;
  dm.aux_stride = aux_stride;
  dm.aux = m->d_aux;
  dm.o2s = m->d_o2s;
  dm.gmap = m->d_gmap;
  dm.olist = m->d_olist;
  dm.gmap_s = m->d_gmap_s;
  dm.gdst = m->d_gdst;
  dm.iel = m->d_iel;
  dm.igrp = m->d_igrp;
  dm.ipt = m->d_ipt;
  // multi-rank buffers
  if (h.nranks > 1) {
    CUDA_TRY(m->alloc(&m->d_send, h.send_list.size()));
    if (!h.send_list.empty())
      CUDA_TRY(cudaMemcpy(m->d_send, h.send_list.data(), h.send_list.size() * 4,
                          cudaMemcpyHostToDevice));
    CUDA_TRY(m->alloc(&m->d_sendbuf, size_t(NF) * h.send_list.size()));
    CUDA_TRY(m->alloc(&m->d_recvbuf, size_t(NF) * h.n_ghost_dof));
    m->po_send.np = m->po_recv.np = h.nranks;
    m->po_send.off[0] = m->po_recv.off[0] = 0;
    for (int p = 0; p < h.nranks; ++p) {
      m->po_send.off[p + 1] = m->po_send.off[p] + h.send_counts[p];
      m->po_recv.off[p + 1] = m->po_recv.off[p] + h.recv_counts[p];
    }
    if (m->po_recv.off[h.nranks] != h.n_ghost_dof || m->po_send.off[h.nranks] != int64_t(h.send_list.size()))
      return fail(DGR_ERR_TREE, "send/receive counts inconsistent with the ghost layer");
  }
  CUDA_TRY(m->alloc(&m->d_cnorm, 16 + size_t(7) * 2 * CN_BLOCKS));   // [16] result + partials
  CUDA_TRY(cudaStreamSynchronize(st));
  return DGR_OK;
}

dgr_status dgr_mesh_create(const dgr_mesh_desc* desc, const dgr_octant* octs, int64_t n,
                           void* stream, dgr_mesh* out) {
  if (!desc || !octs || !out || n <= 0) return fail(DGR_ERR_ARG, "null argument or n <= 0");
  *out = nullptr;
  if (desc->nranks < 1 || desc->nranks > MAX_RANKS || desc->rank < 0 || desc->rank >= desc->nranks)
    return fail(DGR_ERR_ARG, "rank / nranks out of range (1 <= nranks <= 64)");
  std::unique_ptr<dgr_mesh_s> m;
  try {
    m.reset(new dgr_mesh_s());
    std::vector<Oct> leaves(n);
    for (int64_t i = 0; i < n; ++i)
      leaves[i] = {{int64_t(octs[i].x), int64_t(octs[i].y), int64_t(octs[i].z)},
                   int(octs[i].level)};
    m->host.build(desc->xmin, desc->width, desc->max_depth, desc->periodic != 0, leaves,
                  desc->rank, desc->nranks);
  } catch (const BuildError& e) {
    return fail(dgr_status(e.code), e.msg);
  } catch (const std::bad_alloc&) {
    return fail(DGR_ERR_OOM, "host allocation failed");
  }
  for (int k = 0; k < 3; ++k) m->xmin[k] = desc->xmin[k];
  m->device = desc->device != 0;
  if (m->device) {
    dgr_status s = upload(m.get(), static_cast<cudaStream_t>(stream));
    if (s != DGR_OK) return s;
    if (desc->nranks > 1 && desc->nccl_id) {
      // (nccl_id == NULL: external-exchange mode, the caller refreshes ghosts)
      if (!load_nccl()) return fail(DGR_ERR_NCCL, "libnccl.so.2 not loadable");
      UniqueId uid;
      std::memcpy(uid.internal, desc->nccl_id, 128);
      if (g_init_rank(&m->comm, desc->nranks, uid, desc->rank) != 0)
        return fail(DGR_ERR_NCCL, "ncclCommInitRank failed");
    }
  }
  *out = m.release();
  return DGR_OK;
}

dgr_status dgr_mesh_info_get(dgr_mesh m, dgr_mesh_info* info) {
  if (!m || !info) return fail(DGR_ERR_ARG, "null argument");
  const HostMesh& h = m->host;
  info->n_oct_global = int64_t(h.oct.size());
  info->n_oct_local = h.n_owned_oct;
  info->n_oct_ghost = h.n_ghost_oct;
  info->oct_begin = h.oct_begin;
  info->n_dof_global = h.n_dof;
  info->n_dof_owned = h.n_owned_dof;
  info->n_dof_ghost = h.n_ghost_dof;
  const int64_t nd = h.n_owned_dof + h.n_ghost_dof;
  info->dof_stride = ((nd + 31) / 32) * 32;
  info->patch_pitch = PATCH_PITCH;
  info->n_hanging = int64_t(h.hang_rows.size());
  info->level_min = h.level_min;
  info->level_max = h.level_max;
  info->h_min = h.width / (6.0 * std::ldexp(1.0, h.level_max));
  info->n_interp_slots = m->n_interp;
  info->n_interp_elems = m->dm.n_iel;
  info->n_oct_interior = m->device ? m->n_interior : h.n_owned_oct;
  return DGR_OK;
}

dgr_status dgr_mesh_export_maps(dgr_mesh m, int which, void* host_buf, size_t* nbytes) {
  if (!m || !nbytes) return fail(DGR_ERR_ARG, "null argument");
  const HostMesh& h = m->host;
  const int64_t N = int64_t(h.oct.size()), no = h.n_owned_oct;
  std::vector<char> tmp;
  auto put = [&](const void* src, size_t n) -> dgr_status {
    if (!host_buf) {
      *nbytes = n;
      return DGR_OK;
    }
    if (*nbytes < n) return fail(DGR_ERR_ARG, "buffer too small");
    std::memcpy(host_buf, src, n);
    *nbytes = n;
    return DGR_OK;
  };
  switch (which) {
    case DGR_MAP_OCTANTS: {
      std::vector<int32_t> v(4 * N);
      for (int64_t i = 0; i < N; ++i) {
        v[4 * i] = int32_t(h.oct[i].a[0]);
        v[4 * i + 1] = int32_t(h.oct[i].a[1]);
        v[4 * i + 2] = int32_t(h.oct[i].a[2]);
        v[4 * i + 3] = h.oct[i].l;
      }
      return put(v.data(), v.size() * 4);
    }
    case DGR_MAP_O2N:
      return put(h.o2n.data() + size_t(h.oct_begin) * NPT, size_t(no) * NPT * 4);
    case DGR_MAP_HANGING: {
      std::vector<std::array<int32_t, 3>> rows;
      for (const auto& r : h.hang_rows)
        if (r.e_local < no) rows.push_back({r.e_global, r.node, r.src_global});
      std::sort(rows.begin(), rows.end());
      return put(rows.data(), rows.size() * 12);
    }
    case DGR_MAP_PAD_SRC:
      return put(h.pad_src_global.data(), h.pad_src_global.size() * 4);
    case DGR_MAP_PAD_KIND:
      return put(h.pad_kind.data(), h.pad_kind.size());
    case DGR_MAP_ZIP: {
      std::vector<int32_t> v(2 * h.n_owned_dof);
      for (int64_t l = 0; l < h.n_owned_dof; ++l) {
        const int64_t g = h.dof_gid[l];
        v[2 * l] = h.zip_leaf[g];
        v[2 * l + 1] = h.zip_node[g];
      }
      return put(v.data(), v.size() * 4);
    }
    case DGR_MAP_DOF_GID:
      return put(h.dof_gid.data(), h.dof_gid.size() * 8);
    case DGR_MAP_DOF_XYZ: {
      const int64_t nd = int64_t(h.dof_gid.size());
      std::vector<double> v(3 * nd);
      const double unit = h.width / double(h.L);
      for (int64_t d = 0; d < nd; ++d) {
        const int64_t g = h.dof_gid[d];
        const int32_t e = h.zip_leaf[g], n = h.zip_node[g];
        const Oct& o = h.oct[e];
        const int64_t s = h.side(e);
        const int64_t X[3] = {6 * o.a[0] + (n % 7) * s, 6 * o.a[1] + ((n / 7) % 7) * s,
                              6 * o.a[2] + (n / 49) * s};
        for (int k = 0; k < 3; ++k) v[k * nd + d] = h.xmin[k] + double(X[k]) * unit;
      }
      return put(v.data(), v.size() * 8);
    }
    case DGR_MAP_SEND:
      return put(h.send_list.data(), h.send_list.size() * 4);
    case DGR_MAP_SEND_COUNTS:
      return put(h.send_counts.data(), h.send_counts.size() * 8);
    case DGR_MAP_RECV_COUNTS:
      return put(h.recv_counts.data(), h.recv_counts.size() * 8);
    case DGR_MAP_LOCAL_OCTS:
      return put(h.local_oct.data(), h.local_oct.size() * 4);
    case DGR_MAP_O2N_LOCAL:
      return put(h.o2n_local.data(), h.o2n_local.size() * 4);
    case DGR_MAP_SENDBUF: {   // test hook: the last packed (peer-major) send buffer
      if (!m->device) return fail(DGR_ERR_STATE, "send buffer exists on device meshes only");
      const size_t nd = size_t(NF) * h.send_list.size();
      std::vector<double> v(nd);
      if (nd) {
        cudaError_t e = cudaDeviceSynchronize();
        if (e == cudaSuccess) e = cudaMemcpy(v.data(), m->d_sendbuf, nd * 8, cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) return fail(DGR_ERR_CUDA, cudaGetErrorString(e));
      }
      return put(v.data(), v.size() * 8);
    }
    case DGR_MAP_RHS_ORDER: {
      if (!m->device) return fail(DGR_ERR_STATE, "RHS order exists on device meshes only");
      std::vector<int32_t> v(static_cast<size_t>(no));
      if (no) {
        cudaError_t e = cudaMemcpy(v.data(), m->d_olist, size_t(no) * 4, cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) return fail(DGR_ERR_CUDA, cudaGetErrorString(e));
      }
      return put(v.data(), v.size() * 4);
    }
  }
  return fail(DGR_ERR_ARG, "unknown map id");
}

dgr_status dgr_mesh_destroy(dgr_mesh m) {
  if (m && m->group) return fail(DGR_ERR_STATE, "mesh is in a group: dgr_group_destroy first");
  delete m;
  return DGR_OK;
}

int64_t dgr_last_launch_count(dgr_mesh m) { return m ? m->launches : -1; }

}  // extern "C"

// ------------------------------------------------------------- device ops
static dgr_status need_device(dgr_mesh m) {
  if (!m) return fail(DGR_ERR_ARG, "null mesh");
  if (!m->device) return fail(DGR_ERR_STATE, "host-only mesh (desc.device == 0)");
  return DGR_OK;
}

static bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

// Bracket one launch with CUDA events on its stream when profiling is on.
#define PROF(m, cls, st, stmt)                                   \
  do {                                                           \
    cudaEvent_t _a = nullptr;                                    \
    if ((m)->prof) {                                             \
      _a = (m)->ev();                                            \
      cudaEventRecord(_a, (st));                                 \
    }                                                            \
    stmt;                                                        \
    ++(m)->launches;                                             \
    if ((m)->prof) {                                             \
      cudaEvent_t _b = (m)->ev();                                \
      cudaEventRecord(_b, (st));                                 \
      (m)->pend.push_back({(cls), _a, _b});                      \
    }                                                            \
  } while (0)

#define NCCL_TRY(x)                                                                   \
  do {                                                                                \
    int _r = (x);                                                                     \
    if (_r != 0) return fail(DGR_ERR_NCCL, std::string(#x) + " failed: ncclResult " + std::to_string(_r)); \
  } while (0)

// Ghost exchange over NCCL (Alg. 1 line 5 halo_exchange): pack the
// owned DOFs each peer needs into the peer-major send buffer, one grouped
// ncclSend / ncclRecv per peer (a single [NF][n_p] message each way), unpack
// the peer-major receive buffer into u's ghost slice.  All on stream `st`.
static dgr_status exchange(dgr_mesh m, double* u, cudaStream_t st) {
  const HostMesh& h = m->host;
  // single rank; or no communicator: external-exchange / grouped meshes, whose
  // ghosts the caller (DGR_MAP_SEND) or the group driver (dgr_group_*) refreshes
  if (h.nranks <= 1 || !m->comm) return DGR_OK;
  const int64_t stride = m->dm.dof_stride;
  PROF(m, 5, st, launch_gather_pack(u, stride, m->d_send, m->po_send, m->d_sendbuf, st));
  CUDA_TRY(cudaGetLastError());
  NCCL_TRY(g_nccl.GroupStart());
  for (int peer = 0; peer < h.nranks; ++peer) {
    const int64_t ns = h.send_counts[peer], nr = h.recv_counts[peer];
    if (ns) NCCL_TRY(g_nccl.Send(m->d_sendbuf + NF * m->po_send.off[peer], size_t(NF * ns),
                                 NCCL_FLOAT64, peer, m->comm, st));
    if (nr) NCCL_TRY(g_nccl.Recv(m->d_recvbuf + NF * m->po_recv.off[peer], size_t(NF * nr),
                                 NCCL_FLOAT64, peer, m->comm, st));
  }
  NCCL_TRY(g_nccl.GroupEnd());
  PROF(m, 5, st, launch_scatter_unpack(u, stride, h.n_owned_dof, m->d_recvbuf, m->po_recv, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

// interpolation slots (hanging nodes and coarse-neighbour padding values,
// Alg. 2 lines 4-5 and P:L295), one k_interp launch per dependency depth
// (phase 0: slot elements that need owned DOFs only; 1: the rest; -1: both)
static dgr_status do_interp(dgr_mesh m, const double* u, int nf, cudaStream_t st, int phase = -1) {
  for (int ph = 0; ph < 2; ++ph) {
    if (phase >= 0 && ph != phase) continue;
    const std::vector<int64_t>& off = m->iel_depth_off[ph];
    for (size_t g = 0; g + 1 < off.size(); ++g)
      if (off[g + 1] > off[g]) PROF(m, 7, st, launch_interp(m->dm, u, nf, off[g], off[g + 1] - off[g], st));
  }
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

// explicit unzip into the patch buffer (two-pass path, constraints) or straight
// into the caller's buffer (dgr_unzip: same [nf][n_owned][PATCH_PITCH] layout)
static dgr_status do_unzip(dgr_mesh m, const double* u, int nf, cudaStream_t st,
                           double* out = nullptr) {
  if (!out && !m->d_patch) {
    CUDA_TRY(m->alloc(&m->d_patch, size_t(NF) * m->dm.n_owned * PATCH_PITCH));
    CUDA_TRY(cudaMemsetAsync(m->d_patch, 0, size_t(NF) * m->dm.n_owned * PATCH_PITCH * 8, st));
  }
  dgr_status s = do_interp(m, u, nf, st);
  if (s) return s;
  PROF(m, 2, st, launch_unzip(m->dm, u, out ? out : m->d_patch, nf, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

static RhsParams to_rp(const dgr_params* p) {
  RhsParams r{0.4, 2.0, 1.0, 0.0, 1e-4, 0, 0};
  if (p)
    r = {p->ko_sigma, p->eta, p->lambda_f0, p->lambda_f1, p->chi_floor, p->sommerfeld != 0,
         p->upwind != 0};
  return r;
}

// Ghost exchange + RHS of every owned octant's interior points into d_rhs_oct,
// by the fused path (patches gathered inside k_rhs) or through the explicit
// patch buffer.  With a communicator (N > 1) the fused path overlaps the
// exchange with the interior octants: the pack + NCCL group runs
// on its own stream while k_interp (phase 0) and k_rhs work through the
// octants whose patches need no ghost value — k_rhs then leaves a few SMs
// free, since it otherwise holds every SM and the NCCL kernels could not
// start — and the boundary octants follow once the ghosts have landed.
// The fused path without the radiative boundary zips in k_rhs's store
static bool zip_by_store(dgr_mesh m, const dgr_params* prm) {
  (void)prm;   // (the radiative boundary too, since its values are parked in TMEM)
  return m->fused && m->zip_store;
}

static dgr_status ensure_xstream(dgr_mesh m) {
  if (!m->xstream) {
    CUDA_TRY(cudaStreamCreateWithFlags(&m->xstream, cudaStreamNonBlocking));
    CUDA_TRY(cudaEventCreateWithFlags(&m->ev_ready, cudaEventDisableTiming));
    CUDA_TRY(cudaEventCreateWithFlags(&m->ev_xdone, cudaEventDisableTiming));
  }
  return DGR_OK;
}

// (rhs_dof != nullptr: fused path only, k_rhs zips by its store into rhs_dof)
// preissued: the ghost exchange of u was already enqueued on m->xstream by the
// group driver (dgr_group_*) and completes at m->ev_xdone; otherwise it is done
// here (NCCL) — on the caller's stream, or on m->xstream overlapped with the
// interior octants.
// rk (fused path with rhs_dof only): the RK4 stage update fields of RhsParams,
// applied by k_rhs's epilogue instead of storing the RHS
static dgr_status rhs_oct(dgr_mesh m, double* u, const dgr_params* prm, cudaStream_t st,
                          double* rhs_dof = nullptr, bool preissued = false,
                          const RhsParams* rk = nullptr) {
  dgr_status s;
  const int64_t no = m->dm.n_owned, ni = m->n_interior;
  RhsParams rp = to_rp(prm);
  if (rk && rhs_dof) {
    rp.rk_stage = rk->rk_stage;
    rp.rk_dt = rk->rk_dt;
    rp.rk_un = rk->rk_un;
    rp.rk_acc = rk->rk_acc;
    rp.rk_us = rk->rk_us;
    rp.rk_out = rk->rk_out;
  }
  double* pre = nullptr;
  if (m->fused && m->prepass) {
    if (!m->d_pre) CUDA_TRY(m->alloc(&m->d_pre, size_t(pre_rows()) * no * 352));
    pre = m->d_pre;
  }
  // ghosts current on `st` (no overlap)
  auto ghosts_now = [&]() -> dgr_status {
    if (preissued) {
      CUDA_TRY(cudaStreamWaitEvent(st, m->ev_xdone, 0));
      return DGR_OK;
    }
    return exchange(m, u, st);
  };
  if (!m->fused) {
    if ((s = ghosts_now())) return s;
    if ((s = do_unzip(m, u, NF, st))) return s;
    PROF(m, 3, st, launch_rhs(m->dm, m->d_patch, m->d_rhs_oct, rp, false, 0, no, 0, st));
    CUDA_TRY(cudaGetLastError());
    return DGR_OK;
  }
  const bool multi = m->host.nranks > 1 && (m->comm || preissued);
  const bool overlap = multi && ni > 0 && ni < no && m->phases == 0;
  if (m->phases > 0) {
    // interior octants and the slots they need first, then (unless the test
    // hook stops here) the rest — no stream overlap
    if ((s = ghosts_now())) return s;
    if ((s = do_interp(m, u, NF, st, 0))) return s;
    PROF(m, 3, st, launch_rhs(m->dm, u, m->d_rhs_oct, rp, true, 0, ni, 0, st, pre, rhs_dof));
    if (pre) ++m->launches;   // (k_gt_pre + k_rhs)
    if (m->phases == 1) {
      if ((s = do_interp(m, u, NF, st, 1))) return s;
      PROF(m, 3, st, launch_rhs(m->dm, u, m->d_rhs_oct, rp, true, ni, no - ni, 0, st, pre, rhs_dof));
      if (pre) ++m->launches;
    }
  } else if (overlap) {
    if (!preissued) {
      if ((s = ensure_xstream(m))) return s;
      CUDA_TRY(cudaEventRecord(m->ev_ready, st));
      CUDA_TRY(cudaStreamWaitEvent(m->xstream, m->ev_ready, 0));
      if ((s = exchange(m, u, m->xstream))) return s;
      CUDA_TRY(cudaEventRecord(m->ev_xdone, m->xstream));
    }
    if ((s = do_interp(m, u, NF, st, 0))) return s;
    PROF(m, 3, st, launch_rhs(m->dm, u, m->d_rhs_oct, rp, true, 0, ni, m->xsm, st, pre, rhs_dof));
    if (pre) ++m->launches;   // (k_gt_pre + k_rhs)
    CUDA_TRY(cudaStreamWaitEvent(st, m->ev_xdone, 0));
    if ((s = do_interp(m, u, NF, st, 1))) return s;
    PROF(m, 3, st, launch_rhs(m->dm, u, m->d_rhs_oct, rp, true, ni, no - ni, 0, st, pre, rhs_dof));
    if (pre) ++m->launches;
  } else {
    if ((s = ghosts_now())) return s;
    if ((s = do_interp(m, u, NF, st))) return s;
    PROF(m, 3, st, launch_rhs(m->dm, u, m->d_rhs_oct, rp, true, 0, no, 0, st, pre, rhs_dof));
    if (pre) ++m->launches;   // (k_gt_pre + k_rhs)
  }
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

extern "C" {

dgr_status dgr_dof_coords(dgr_mesh m, double* xyz, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!xyz) return fail(DGR_ERR_ARG, "null xyz");
  launch_dof_coords(m->dm, m->d_dof_node, xyz, m->xmin, static_cast<cudaStream_t>(stream));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

dgr_status dgr_ghost_exchange(dgr_mesh m, double* u, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (m->host.nranks > 1 && !m->comm)
    return fail(DGR_ERR_STATE, "external-exchange mesh (created without nccl_id)");
  return exchange(m, u, static_cast<cudaStream_t>(stream));
}

dgr_status dgr_unzip(dgr_mesh m, const double* u, double* patches, int nfields, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!u || !patches || nfields < 1 || nfields > NF) return fail(DGR_ERR_ARG, "bad unzip args");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  m->launches = 0;
  if (!aligned16(patches)) return fail(DGR_ERR_ARG, "patches must be 16-byte aligned");
  return do_unzip(m, u, nfields, st, patches);
}

dgr_status dgr_rhs_patches(dgr_mesh m, const double* patches, double* rhs_oct,
                           const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!patches || !rhs_oct || !aligned16(patches)) return fail(DGR_ERR_ARG, "bad rhs args");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  PROF(m, 3, st, launch_rhs(m->dm, patches, rhs_oct, to_rp(prm), false, 0, m->dm.n_owned, 0, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

dgr_status dgr_rhs(dgr_mesh m, double* u, double* rhs, const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!u || !rhs) return fail(DGR_ERR_ARG, "null state");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  m->launches = 0;
  if (zip_by_store(m, prm)) return rhs_oct(m, u, prm, st, rhs);
  if ((s = rhs_oct(m, u, prm, st))) return s;
  PROF(m, 4, st, launch_zip(m->dm, m->d_rhs_oct, rhs, NF, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

// u_s: the previous stage's state (gathered by stages 1-3); u_s_next (fused
// RK4 update only, != u_s): where this stage writes its state
static dgr_status stage(dgr_mesh m, int s_, double dt, double* u_n, double* u_s, double* acc,
                        double* u_out, const dgr_params* prm, cudaStream_t st,
                        bool preissued = false, double* u_s_next = nullptr) {
  dgr_status s;
  double* cur = s_ == 0 ? u_n : u_s;
  if (u_s_next && zip_by_store(m, prm)) {
    if (!m->d_rhs_dof) CUDA_TRY(m->alloc(&m->d_rhs_dof, size_t(NF) * m->dm.dof_stride));
    RhsParams rk = to_rp(prm);
    rk.rk_stage = s_;
    rk.rk_dt = dt;
    rk.rk_un = u_n;
    rk.rk_acc = acc;
    rk.rk_us = u_s_next;
    rk.rk_out = u_out;
    if ((s = rhs_oct(m, cur, prm, st, m->d_rhs_dof, preissued, &rk))) return s;
    CUDA_TRY(cudaGetLastError());
    return DGR_OK;
  }
  // (applying the zip + RK4 update inside k_rhs measured 10.6 ms vs 7.5 + 0.8 ms
  // for RHS + k_zip_rk4 on C3 — the scattered state loads stall the single
  // persistent CTA per SM — so the update is a separate kernel; the zip itself
  // is only stores, so k_rhs does it by default: DGR_OPT_ZIP_STORE)
  if (zip_by_store(m, prm)) {
    if (!m->d_rhs_dof) CUDA_TRY(m->alloc(&m->d_rhs_dof, size_t(NF) * m->dm.dof_stride));
    if ((s = rhs_oct(m, cur, prm, st, m->d_rhs_dof, preissued))) return s;
    PROF(m, 4, st, launch_rk4(m->dm, m->d_rhs_dof, s_, dt, u_n, u_s, acc, u_out, st));
    CUDA_TRY(cudaGetLastError());
    return DGR_OK;
  }
  if ((s = rhs_oct(m, cur, prm, st, nullptr, preissued))) return s;
  PROF(m, 4, st, launch_zip_rk4(m->dm, m->d_rhs_oct, s_, dt, u_n, u_s, acc, u_out, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

// the four stages of one RK4 step of u (in place), with the fused update
// (DGR_OPT_FUSE_RK4) when the path allows it: stage k gathers u, d_us, d_us2,
// d_us and writes d_us, d_us2, d_us, u
static dgr_status four_stages(dgr_mesh m, double dt, double* u, const dgr_params* prm,
                              cudaStream_t q) {
  const bool fz = m->fuse_rk4 && zip_by_store(m, prm);
  if (fz && !m->d_us2) {
    CUDA_TRY(m->alloc(&m->d_us2, size_t(NF) * m->dm.dof_stride));
    CUDA_TRY(cudaMemset(m->d_us2, 0, size_t(NF) * m->dm.dof_stride * 8));
  }
  for (int k = 0; k < 4; ++k) {
    double* in = k == 2 && fz ? m->d_us2 : m->d_us;
    double* out = fz ? (k == 1 ? m->d_us2 : m->d_us) : nullptr;
    if (dgr_status e = stage(m, k, dt, u, in, m->d_acc, u, prm, q, false, out)) return e;
  }
  return DGR_OK;
}

dgr_status dgr_rk4_stage(dgr_mesh m, int s_, double dt, double* u_n, double* u_s, double* acc,
                         const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (s_ < 0 || s_ > 3 || !u_n || !u_s || !acc) return fail(DGR_ERR_ARG, "bad stage args");
  m->launches = 0;
  return stage(m, s_, dt, u_n, u_s, acc, acc, prm, static_cast<cudaStream_t>(stream));
}

static bool same_key(const dgr_mesh_s::GraphKey& a, const dgr_mesh_s::GraphKey& b) {
  return a.u == b.u && std::memcmp(&a.dt, &b.dt, sizeof(double)) == 0 && a.has_prm == b.has_prm &&
         (!a.has_prm || std::memcmp(&a.prm, &b.prm, sizeof(dgr_params)) == 0);
}

dgr_status dgr_rk4_step(dgr_mesh m, double dt, double* u, const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!u) return fail(DGR_ERR_ARG, "null state");
  if (m->host.nranks > 1 && !m->comm)
    return fail(DGR_ERR_STATE, "dgr_rk4_step needs a communicator: external-exchange meshes step "
                               "with dgr_rk4_stage, grouped meshes with dgr_group_rk4_step");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  auto eager = [&](cudaStream_t q) -> dgr_status {
    m->launches = 0;
    return four_stages(m, dt, u, prm, q);
  };
  // CUDA graph of the step (the 16+ launches of the 4 stages, and with N > 1
  // the exchange stream's pack / NCCL / unpack, captured once): the first call
  // with given arguments runs eagerly (lazy allocations happen there), the
  // second captures on a library stream and instantiates, later calls replay.
  // Profiling (per-launch events) and NCCL meshes run eagerly.
  if (!m->use_graph || m->prof || m->comm) return eager(st);
  dgr_mesh_s::GraphKey key{u, dt, prm ? *prm : dgr_params{}, prm != nullptr};
  if (!same_key(key, m->gkey)) {
    m->drop_graph();
    m->gkey = key;
  }
  if (m->gseen++ == 0) return eager(st);
  if (!m->gexec) {
    if (!m->gstream) CUDA_TRY(cudaStreamCreateWithFlags(&m->gstream, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamBeginCapture(m->gstream, cudaStreamCaptureModeThreadLocal));
    dgr_status e = eager(m->gstream);
    cudaGraph_t graph = nullptr;
    cudaError_t ce = cudaStreamEndCapture(m->gstream, &graph);
    if (e) {
      if (graph) cudaGraphDestroy(graph);
      return e;
    }
    CUDA_TRY(ce);
    ce = cudaGraphInstantiate(&m->gexec, graph, 0);
    cudaGraphDestroy(graph);
    CUDA_TRY(ce);
    m->glaunches = m->launches;
  }
  CUDA_TRY(cudaGraphLaunch(m->gexec, st));
  m->launches = m->glaunches;
  return DGR_OK;
}

// n independent host-resident states, one RK4 step each, through three device
// slots: the H2D copy of state j+1 (h2d stream) and the D2H copy of state j-1
// (d2h stream) run on the copy engines while state j steps on `stream`.
// Slot b = j % 3 is reused by state j+3 only after state j's D2H completed.
dgr_status dgr_rk4_step_host(dgr_mesh m, double dt, int64_t n, const double* const* u_in,
                             double* const* u_out, const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (n < 0 || (n > 0 && (!u_in || !u_out))) return fail(DGR_ERR_ARG, "bad host state lists");
  for (int64_t j = 0; j < n; ++j)
    if (!u_in[j] || !u_out[j]) return fail(DGR_ERR_ARG, "null host state");
  if (m->host.nranks > 1 && !m->comm)
    return fail(DGR_ERR_STATE, "dgr_rk4_step_host needs a communicator (the stages refresh the "
                               "ghost DOFs by NCCL)");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  m->launches = 0;
  if (n == 0) return DGR_OK;
  const int64_t stride = m->dm.dof_stride;
  const size_t pitch = size_t(stride) * 8;
  const size_t width = size_t(m->host.n_owned_dof) * 8;   // ghosts come from the exchange
  const int nb = n < 3 ? int(n) : 3;
  for (int b = 0; b < nb; ++b)
    if (!m->d_hbuf[b]) {
      CUDA_TRY(m->alloc(&m->d_hbuf[b], size_t(NF) * stride));
      CUDA_TRY(cudaMemset(m->d_hbuf[b], 0, size_t(NF) * pitch));   // ghost rows defined
    }
  if (!m->h2d) {
    CUDA_TRY(cudaStreamCreateWithFlags(&m->h2d, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamCreateWithFlags(&m->d2h, cudaStreamNonBlocking));
    CUDA_TRY(cudaEventCreateWithFlags(&m->ev_host0, cudaEventDisableTiming));
    for (int b = 0; b < 3; ++b) {
      CUDA_TRY(cudaEventCreateWithFlags(&m->ev_in[b], cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&m->ev_done[b], cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&m->ev_out[b], cudaEventDisableTiming));
    }
  }
  // the copy streams start after the work already on the caller's stream
  CUDA_TRY(cudaEventRecord(m->ev_host0, st));
  CUDA_TRY(cudaStreamWaitEvent(m->h2d, m->ev_host0, 0));
  CUDA_TRY(cudaStreamWaitEvent(m->d2h, m->ev_host0, 0));
  for (int64_t j = 0; j < n; ++j) {
    const int b = int(j % 3);
    double* ub = m->d_hbuf[b];
    if (j >= 3) CUDA_TRY(cudaStreamWaitEvent(m->h2d, m->ev_out[b], 0));
    CUDA_TRY(cudaMemcpy2DAsync(ub, pitch, u_in[j], pitch, width, NF, cudaMemcpyHostToDevice,
                               m->h2d));
    CUDA_TRY(cudaEventRecord(m->ev_in[b], m->h2d));
    CUDA_TRY(cudaStreamWaitEvent(st, m->ev_in[b], 0));
    if ((s = four_stages(m, dt, ub, prm, st))) return s;   // (launch counts accumulate)
    CUDA_TRY(cudaEventRecord(m->ev_done[b], st));
    CUDA_TRY(cudaStreamWaitEvent(m->d2h, m->ev_done[b], 0));
    CUDA_TRY(cudaMemcpy2DAsync(u_out[j], pitch, ub, pitch, width, NF, cudaMemcpyDeviceToHost,
                               m->d2h));
    CUDA_TRY(cudaEventRecord(m->ev_out[b], m->d2h));
  }
  // the caller's stream completes after the last D2H copy
  CUDA_TRY(cudaStreamWaitEvent(st, m->ev_out[(n - 1) % 3], 0));
  return DGR_OK;
}

dgr_status dgr_constraints(dgr_mesh m, double* u, double* c, double* norms_host,
                           const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!u || !c) return fail(DGR_ERR_ARG, "null argument");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  m->launches = 0;
  if ((s = exchange(m, u, st))) return s;
  if ((s = do_unzip(m, u, NF, st))) return s;
  PROF(m, 6, st, launch_constraints(m->dm, m->d_patch, m->d_rhs_oct, to_rp(prm), st));
  CUDA_TRY(cudaGetLastError());
  // zip the 7 constraint fields
  const int64_t stride = m->dm.dof_stride;
  DevMesh dm = m->dm;
  PROF(m, 4, st, launch_zip(dm, m->d_rhs_oct, c, 7, st));
  CUDA_TRY(cudaGetLastError());
  if (norms_host) {
    // norms on the device (deterministic two-pass reduction), 14 doubles to the host
    const int64_t n = m->host.n_owned_dof;
    PROF(m, 6, st, launch_cnorms(c, stride, n, 7, m->d_cnorm + 16, m->d_cnorm, st));
    CUDA_TRY(cudaGetLastError());
    double part[14];
    CUDA_TRY(cudaMemcpyAsync(part, m->d_cnorm, sizeof(part), cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    double ntot = double(n);
    if (m->host.nranks > 1 && m->comm) {   // (external-exchange mode: rank-local norms)
      double* d = m->d_cnorm;
      double sums[8], maxs[7];
      for (int q = 0; q < 7; ++q) {
        sums[q] = part[2 * q];
        maxs[q] = part[2 * q + 1];
      }
      sums[7] = ntot;
      CUDA_TRY(cudaMemcpyAsync(d, sums, 64, cudaMemcpyHostToDevice, st));
      CUDA_TRY(cudaMemcpyAsync(d + 8, maxs, 56, cudaMemcpyHostToDevice, st));
      NCCL_TRY(g_nccl.AllReduce(d, d, 8, NCCL_FLOAT64, NCCL_SUM, m->comm, st));
      NCCL_TRY(g_nccl.AllReduce(d + 8, d + 8, 7, NCCL_FLOAT64, NCCL_MAX, m->comm, st));
      CUDA_TRY(cudaMemcpyAsync(sums, d, 64, cudaMemcpyDeviceToHost, st));
      CUDA_TRY(cudaMemcpyAsync(maxs, d + 8, 56, cudaMemcpyDeviceToHost, st));
      CUDA_TRY(cudaStreamSynchronize(st));
      for (int q = 0; q < 7; ++q) {
        part[2 * q] = sums[q];
        part[2 * q + 1] = maxs[q];
      }
      ntot = sums[7];
    }
    for (int q = 0; q < 7; ++q) {
      norms_host[2 * q] = std::sqrt(part[2 * q] / std::max(ntot, 1.0));
      norms_host[2 * q + 1] = part[2 * q + 1];
    }
  }
  return DGR_OK;
}

dgr_status dgr_rhs_inputs(dgr_mesh m, double* u, double* in, int64_t ld, const dgr_params* prm,
                          void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  const int64_t n = int64_t(m->dm.n_owned) * NPT;
  if (!u || !in || ld < n) return fail(DGR_ERR_ARG, "bad rhs_inputs args (ld >= n_oct_local * 343)");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  m->launches = 0;
  if ((s = exchange(m, u, st))) return s;
  if ((s = do_unzip(m, u, NF, st))) return s;
  const RhsParams rp = to_rp(prm);
  PROF(m, 3, st, launch_rhs_inputs(m->dm, m->d_patch, in, ld, rp.ko_sigma, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

dgr_status dgr_rhs_algebra(int variant, int occ, const double* in, double* out, int64_t n,
                           int64_t ld, const dgr_params* prm, void* stream) {
  if (variant < 0 || variant > 2 || !in || !out || n < 0 || ld < n)
    return fail(DGR_ERR_ARG, "bad rhs_algebra args (variant 0..2, ld >= n)");
  const RhsParams rp = to_rp(prm);
  const AlgParams ap{rp.eta, rp.lambda_f0, rp.lambda_f1, rp.chi_floor};
  launch_rhs_alg(variant, occ ? 1 : 0, in, out, n, ld, ap, static_cast<cudaStream_t>(stream));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

// ------------------------------------------------------------------ regrid
dgr_status dgr_regrid_indicator(dgr_mesh m, double* u, uint32_t field_mask, double* w,
                                void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!u || !w || !(field_mask & 0xffffffu)) return fail(DGR_ERR_ARG, "bad regrid_indicator args");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  m->launches = 0;
  if ((s = exchange(m, u, st))) return s;
  if ((s = do_unzip(m, u, NF, st))) return s;
  PROF(m, 2, st, launch_wavelet(m->dm, m->d_patch, field_mask & 0xffffffu, w, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

dgr_status dgr_regrid_octree(dgr_mesh m, const double* w, double eps_refine, double eps_coarsen,
                             int level_min, int level_max, dgr_octant* out, int64_t* n_inout) {
  if (!m || !w || !n_inout) return fail(DGR_ERR_ARG, "null argument");
  const HostMesh& h = m->host;
  if (level_min < 0 || level_max > h.D || level_min > level_max || !(eps_coarsen <= eps_refine))
    return fail(DGR_ERR_ARG, "bad regrid levels or tolerances (eps_coarsen <= eps_refine)");
  try {
    std::vector<Oct> o = regrid_leaves(h.oct, w, eps_refine, eps_coarsen, level_min, level_max,
                                       h.D, h.periodic);
    if (!out) {
      *n_inout = int64_t(o.size());
      return DGR_OK;
    }
    if (*n_inout < int64_t(o.size())) return fail(DGR_ERR_ARG, "output buffer too small");
    for (size_t i = 0; i < o.size(); ++i)
      out[i] = {uint32_t(o[i].a[0]), uint32_t(o[i].a[1]), uint32_t(o[i].a[2]), uint32_t(o[i].l)};
    *n_inout = int64_t(o.size());
    return DGR_OK;
  } catch (const std::bad_alloc&) {
    return fail(DGR_ERR_OOM, "host allocation failed");
  }
}

dgr_status dgr_regrid_transfer(dgr_mesh old_m, double* u_old, dgr_mesh new_m, double* u_new,
                               void* stream) {
  dgr_status s;
  if ((s = need_device(old_m)) || (s = need_device(new_m))) return s;
  if (!u_old || !u_new) return fail(DGR_ERR_ARG, "null state");
  const HostMesh& ho = old_m->host;
  const HostMesh& hn = new_m->host;
  if (ho.nranks != 1 || hn.nranks != 1)
    return fail(DGR_ERR_STATE, "dgr_regrid_transfer: single-rank meshes only");
  if (ho.D != hn.D || ho.periodic != hn.periodic || ho.width != hn.width ||
      ho.xmin[0] != hn.xmin[0] || ho.xmin[1] != hn.xmin[1] || ho.xmin[2] != hn.xmin[2])
    return fail(DGR_ERR_ARG, "meshes of different domains");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  // new DOF -> (finest old leaf containing it, lowest Morton index on ties;
  // its half-grid coordinates t2), reading R32
  const int64_t nd = hn.n_owned_dof;
  std::vector<int4> map(size_t(std::max<int64_t>(nd, 1)));
  const int64_t L = ho.L;
  for (int64_t d = 0; d < nd; ++d) {
    const int64_t g = hn.dof_gid[d];
    const int32_t e = hn.zip_leaf[g], n = hn.zip_node[g];
    const Oct& o = hn.oct[e];
    const int64_t sn = hn.side(e);
    const int64_t X[3] = {6 * o.a[0] + (n % 7) * sn, 6 * o.a[1] + ((n / 7) % 7) * sn,
                          6 * o.a[2] + (n / 49) * sn};
    int32_t best = -1;
    for (int q = 0; q < 8; ++q) {
      int64_t c[3];
      for (int a = 0; a < 3; ++a) {
        const int64_t v = 2 * X[a] + (((q >> a) & 1) ? 1 : -1);
        c[a] = v >= 0 ? v / 12 : -((-v + 11) / 12);   // floor division
      }
      const int32_t leaf = ho.locate(c[0], c[1], c[2]);
      if (leaf < 0) continue;
      if (best < 0 || ho.oct[leaf].l > ho.oct[best].l ||
          (ho.oct[leaf].l == ho.oct[best].l && leaf < best))
        best = leaf;
    }
    if (best < 0) return fail(DGR_ERR_TREE, "new DOF outside the old mesh");
    const int64_t so = ho.side(best);
    int t2[3];
    for (int a = 0; a < 3; ++a) {
      int64_t off = X[a] - 6 * ho.oct[best].a[a];
      if (ho.periodic) off = ((off % L) + L) % L;
      if ((2 * off) % so != 0 || 2 * off / so > 12)
        return fail(DGR_ERR_TREE, "new DOF not on the half-grid of its old element "
                                  "(levels changed by more than one)");
      t2[a] = int(2 * off / so);
    }
    const int32_t el = ho.g2l_oct[best];
    map[size_t(d)] = make_int4(el, t2[0] | (t2[1] << 8) | (t2[2] << 16), 0, 0);
  }
  int4* d_map = nullptr;
  CUDA_TRY(cudaMallocAsync(&d_map, map.size() * sizeof(int4), st));
  CUDA_TRY(cudaMemcpyAsync(d_map, map.data(), map.size() * sizeof(int4), cudaMemcpyHostToDevice, st));
  old_m->launches = 0;
  if ((s = do_interp(old_m, u_old, NF, st))) return s;   // hanging-node slots of the old mesh
  PROF(old_m, 2, st, launch_transfer(old_m->dm, u_old, d_map, nd, u_new, new_m->dm.dof_stride, st));
  CUDA_TRY(cudaGetLastError());
  CUDA_TRY(cudaFreeAsync(d_map, st));
  CUDA_TRY(cudaStreamSynchronize(st));   // the host map is freed on return
  return DGR_OK;
}

// ---------------------------------------------------------- Psi_4 extraction
dgr_status dgr_psi4(dgr_mesh m, double* u, const double* center, double* psi,
                    const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!u || !center || !psi) return fail(DGR_ERR_ARG, "null argument");
  const int64_t n = int64_t(m->dm.n_owned) * NPT;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (!m->d_psi_in) CUDA_TRY(m->alloc(&m->d_psi_in, size_t(234) * std::max<int64_t>(n, 1)));
  if (!m->d_psi_xyz) CUDA_TRY(m->alloc(&m->d_psi_xyz, size_t(3) * std::max<int64_t>(n, 1)));
  m->launches = 0;
  if ((s = exchange(m, u, st))) return s;
  if ((s = do_unzip(m, u, NF, st))) return s;
  const RhsParams rp = to_rp(prm);
  const AlgParams ap{rp.eta, rp.lambda_f0, rp.lambda_f1, rp.chi_floor};
  PROF(m, 6, st, launch_rhs_inputs(m->dm, m->d_patch, m->d_psi_in, n, rp.ko_sigma, st));
  PROF(m, 6, st, launch_octant_xyz(m->dm, center, m->d_psi_xyz, n, st));
  PROF(m, 6, st, launch_psi4(m->d_psi_in, m->d_psi_xyz, psi, n, n, ap, st));
  CUDA_TRY(cudaGetLastError());
  return DGR_OK;
}

dgr_status dgr_psi4_sphere(dgr_mesh m, const double* psi, int64_t npts, const double* xyz,
                           double* out, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!psi || npts < 0 || (npts > 0 && (!xyz || !out))) return fail(DGR_ERR_ARG, "bad psi4_sphere args");
  const HostMesh& h = m->host;
  if (h.nranks != 1) return fail(DGR_ERR_STATE, "dgr_psi4_sphere: single-rank meshes only");
  if (npts == 0) return DGR_OK;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const double unit = h.width / double(h.L);
  std::vector<int32_t> oc(static_cast<size_t>(npts));
  std::vector<double> t(static_cast<size_t>(3 * npts));
  for (int64_t k = 0; k < npts; ++k) {
    double X[3];
    int64_t lo[3];
    bool on[3];
    for (int a = 0; a < 3; ++a) {
      X[a] = (xyz[a * npts + k] - h.xmin[a]) / unit;
      lo[a] = int64_t(std::floor(X[a] / 6.0));
      on[a] = double(lo[a]) * 6.0 == X[a];
    }
    // finest leaf whose closed box contains X, lowest Morton index on ties (R36)
    int32_t best = -1;
    for (int q = 0; q < 8; ++q) {
      int64_t c[3];
      for (int a = 0; a < 3; ++a) c[a] = (on[a] && ((q >> a) & 1)) ? lo[a] - 1 : lo[a];
      const int32_t leaf = h.locate(c[0], c[1], c[2]);
      if (leaf < 0) continue;
      if (best < 0 || h.oct[leaf].l > h.oct[best].l ||
          (h.oct[leaf].l == h.oct[best].l && leaf < best))
        best = leaf;
    }
    if (best < 0) return fail(DGR_ERR_ARG, "extraction point outside the domain");
    oc[size_t(k)] = best;
    const double sd = double(h.side(best));
    for (int a = 0; a < 3; ++a) t[size_t(a * npts + k)] = (X[a] - 6.0 * double(h.oct[best].a[a])) / sd;
  }
  int32_t* d_oc = nullptr;
  double *d_t = nullptr, *d_out = nullptr;
  CUDA_TRY(cudaMallocAsync(&d_oc, size_t(npts) * 4, st));
  CUDA_TRY(cudaMallocAsync(&d_t, size_t(3 * npts) * 8, st));
  CUDA_TRY(cudaMallocAsync(&d_out, size_t(2 * npts) * 8, st));
  CUDA_TRY(cudaMemcpyAsync(d_oc, oc.data(), size_t(npts) * 4, cudaMemcpyHostToDevice, st));
  CUDA_TRY(cudaMemcpyAsync(d_t, t.data(), size_t(3 * npts) * 8, cudaMemcpyHostToDevice, st));
  PROF(m, 6, st, launch_sphere_interp(psi, int64_t(m->dm.n_owned) * NPT, d_oc, d_t, npts, d_out, st));
  CUDA_TRY(cudaGetLastError());
  CUDA_TRY(cudaMemcpyAsync(out, d_out, size_t(2 * npts) * 8, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaFreeAsync(d_oc, st));
  CUDA_TRY(cudaFreeAsync(d_t, st));
  CUDA_TRY(cudaFreeAsync(d_out, st));
  CUDA_TRY(cudaStreamSynchronize(st));
  return DGR_OK;
}

// Gauss-Legendre nodes (ascending) and weights by Newton iteration on P_n
static void gauss_legendre(int n, std::vector<double>& x, std::vector<double>& w) {
  x.assign(size_t(n), 0.0);
  w.assign(size_t(n), 0.0);
  for (int i = 0; i < n; ++i) {
    double z = std::cos(M_PI * (i + 0.75) / (n + 0.5)), dp = 0.0;
    for (int it = 0; it < 100; ++it) {
      double p0 = 1.0, p1 = z;
      for (int k = 2; k <= n; ++k) {
        const double p2 = ((2.0 * k - 1.0) * z * p1 - (k - 1.0) * p0) / k;
        p0 = p1;
        p1 = p2;
      }
      if (n == 1) { p1 = z; p0 = 1.0; }
      dp = n * (z * p1 - p0) / (z * z - 1.0);
      const double dz = p1 / dp;
      z -= dz;
      if (std::fabs(dz) < 1e-16) break;
    }
    x[size_t(n - 1 - i)] = z;
    w[size_t(n - 1 - i)] = 2.0 / ((1.0 - z * z) * dp * dp);
  }
}

// spin-weighted spherical harmonic sY_lm (Goldberg et al. 1967), real and
// imaginary parts
static void swsh(int sw, int l, int mm, double th, double ph, double* re, double* im) {
  auto fact = [](int k) { double f = 1.0; for (int i = 2; i <= k; ++i) f *= i; return f; };
  auto comb = [&](int a, int b) { return (b < 0 || b > a) ? 0.0 : fact(a) / (fact(b) * fact(a - b)); };
  if (l < std::abs(sw) || l < std::abs(mm)) { *re = *im = 0.0; return; }
  const double pre = ((mm & 1) ? -1.0 : 1.0) *
                     std::sqrt((2 * l + 1) / (4 * M_PI) * fact(l + mm) * fact(l - mm) /
                               (fact(l + sw) * fact(l - sw)));
  double tot = 0.0;
  for (int r = 0; r <= l - sw; ++r) {
    const int k = r + sw - mm;
    if (k < 0 || k > l + sw) continue;
    tot += comb(l - sw, r) * comb(l + sw, k) * (((l - r - sw) & 1) ? -1.0 : 1.0) *
           std::pow(std::cos(th / 2), 2 * r + sw - mm) * std::pow(std::sin(th / 2), 2 * l - 2 * r - sw + mm);
  }
  *re = pre * tot * std::cos(mm * ph);
  *im = pre * tot * std::sin(mm * ph);
}

dgr_status dgr_psi4_modes(dgr_mesh m, double* u, const double* center, double radius, int n_theta,
                          int n_phi, int l_max, double* modes, double* sphere,
                          const dgr_params* prm, void* stream) {
  dgr_status s = need_device(m);
  if (s) return s;
  if (!u || !center || !modes || radius <= 0 || n_theta < 1 || n_phi < 1 || l_max < 2 || l_max > 12)
    return fail(DGR_ERR_ARG, "bad psi4_modes args (radius > 0, l_max in 2..12)");
  const int64_t n = int64_t(m->dm.n_owned) * NPT;
  if (!m->d_psi) CUDA_TRY(m->alloc(&m->d_psi, size_t(2) * std::max<int64_t>(n, 1)));
  if ((s = dgr_psi4(m, u, center, m->d_psi, prm, stream))) return s;
  std::vector<double> gx, gw;
  gauss_legendre(n_theta, gx, gw);
  const int64_t np = int64_t(n_theta) * n_phi;
  std::vector<double> xyz(static_cast<size_t>(3 * np)), th(static_cast<size_t>(np)),
      ph(static_cast<size_t>(np)), wt(static_cast<size_t>(np));
  for (int i = 0; i < n_theta; ++i)
    for (int j = 0; j < n_phi; ++j) {
      const int64_t k = int64_t(i) * n_phi + j;
      th[size_t(k)] = std::acos(gx[size_t(i)]);
      ph[size_t(k)] = 2.0 * M_PI * j / n_phi;
      wt[size_t(k)] = gw[size_t(i)] * (2.0 * M_PI / n_phi);
      xyz[size_t(k)] = radius * std::sin(th[size_t(k)]) * std::cos(ph[size_t(k)]) + center[0];
      xyz[size_t(np + k)] = radius * std::sin(th[size_t(k)]) * std::sin(ph[size_t(k)]) + center[1];
      xyz[size_t(2 * np + k)] = radius * std::cos(th[size_t(k)]) + center[2];
    }
  std::vector<double> val(static_cast<size_t>(2 * np));
  if ((s = dgr_psi4_sphere(m, m->d_psi, np, xyz.data(), val.data(), stream))) return s;
  if (sphere) std::memcpy(sphere, val.data(), val.size() * 8);
  int q = 0;
  for (int l = 2; l <= l_max; ++l)
    for (int mm = -l; mm <= l; ++mm, ++q) {
      double cr = 0.0, ci = 0.0;
      for (int64_t k = 0; k < np; ++k) {
        double yr, yi;
        swsh(-2, l, mm, th[size_t(k)], ph[size_t(k)], &yr, &yi);
        const double pr = val[size_t(k)], pi_ = val[size_t(np + k)];
        // psi * conj(Y)
        cr += wt[size_t(k)] * (pr * yr + pi_ * yi);
        ci += wt[size_t(k)] * (pi_ * yr - pr * yi);
      }
      modes[2 * q] = cr;
      modes[2 * q + 1] = ci;
    }
  return DGR_OK;
}

dgr_status dgr_set_option(dgr_mesh m, int option, int64_t value) {
  if (!m) return fail(DGR_ERR_ARG, "null mesh");
  switch (option) {
    case DGR_OPT_GRAPH: m->use_graph = value != 0; m->drop_graph(); return DGR_OK;
    case DGR_OPT_FUSE_RK4: m->fuse_rk4 = value != 0; m->drop_graph(); return DGR_OK;
    case DGR_OPT_FUSED_UNZIP: m->fused = value != 0; m->drop_graph(); return DGR_OK;
    case DGR_OPT_PREPASS: m->prepass = value != 0; m->drop_graph(); return DGR_OK;
    case DGR_OPT_ZIP_STORE: m->zip_store = value != 0; m->drop_graph(); return DGR_OK;
    case DGR_OPT_PHASES:
      if (value < 0 || value > 2) return fail(DGR_ERR_ARG, "DGR_OPT_PHASES is 0, 1 or 2");
      m->phases = int(value);
      m->drop_graph();
      return DGR_OK;
  }
  return fail(DGR_ERR_ARG, "unknown option");
}

dgr_status dgr_profile_enable(dgr_mesh m, int on) {
  if (!m) return fail(DGR_ERR_ARG, "null mesh");
  m->prof = on != 0;
  m->drop_graph();
  return DGR_OK;
}

dgr_status dgr_profile_read(dgr_mesh m, double* ms, int64_t* counts, int reset) {
  if (!m) return fail(DGR_ERR_ARG, "null mesh");
  for (auto& p : m->pend) {
    CUDA_TRY(cudaEventSynchronize(p.b));
    float t = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&t, p.a, p.b));
    m->prof_ms[p.cls] += double(t);
    m->prof_n[p.cls] += 1;
    m->pool.push_back(p.a);
    m->pool.push_back(p.b);
  }
  m->pend.clear();
  for (int c = 0; c < DGR_PROF_CLASSES; ++c) {
    if (ms) ms[c] = m->prof_ms[c];
    if (counts) counts[c] = m->prof_n[c];
    if (reset) {
      m->prof_ms[c] = 0;
      m->prof_n[c] = 0;
    }
  }
  return DGR_OK;
}

dgr_status dgr_bench_dfma(int blocks, int iters, void* stream, double* ms, double* flops) {
  if (blocks <= 0 || iters <= 0 || !ms || !flops) return fail(DGR_ERR_ARG, "bad dfma args");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  double* out = nullptr;
  CUDA_TRY(cudaMalloc(&out, 8));
  cudaEvent_t a, b;
  CUDA_TRY(cudaEventCreate(&a));
  CUDA_TRY(cudaEventCreate(&b));
  launch_dfma(blocks, 16, out, st);  // warm-up
  CUDA_TRY(cudaEventRecord(a, st));
  launch_dfma(blocks, iters, out, st);
  CUDA_TRY(cudaEventRecord(b, st));
  CUDA_TRY(cudaEventSynchronize(b));
  float t = 0.f;
  CUDA_TRY(cudaEventElapsedTime(&t, a, b));
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(out);
  *ms = double(t);
  *flops = double(blocks) * 256.0 * 8.0 * double(iters) * 2.0;
  return DGR_OK;
}

}  // extern "C"

// ------------------------------------------------------- in-process rank group
// R rank-meshes of one octree driven by one process (one per device, or several
// on one device).  The exchange is libdgr's own: k_pack into each rank's
// peer-major send buffer, one peer copy per (rank, peer) pair into the peer's
// receive buffer (cudaMemcpyPeerAsync: NVLink between devices, a device copy
// on one device), k_unpack into the ghost slice — the same buffers, offsets and
// kernels as the NCCL path, with the transport replaced.
struct dgr_group_s {
  std::vector<dgr_mesh> m;
  std::vector<cudaEvent_t> ev_packed;   // per rank: its send buffer is packed
  ~dgr_group_s() {
    for (auto e : ev_packed) if (e) cudaEventDestroy(e);
    for (dgr_mesh x : m) if (x && x->group == this) x->group = nullptr;
  }
};

namespace {
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) { cudaGetDevice(&prev); if (d >= 0 && d != prev) cudaSetDevice(d); }
  ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
};
}  // namespace

// enqueue the exchange of every rank's state u[r]; rank r's ghosts are current
// at m[r]->ev_xdone (recorded on m[r]->xstream).  Work starts after what is
// already enqueued on streams[r].
static dgr_status group_exchange(dgr_group_s* g, double* const* u, void* const* streams) {
  const int R = int(g->m.size());
  for (int r = 0; r < R; ++r) {
    dgr_mesh m = g->m[r];
    DeviceGuard dg(m->dev_id);
    cudaStream_t st = static_cast<cudaStream_t>(streams[r]);
    dgr_status s = ensure_xstream(m);
    if (s) return s;
    CUDA_TRY(cudaEventRecord(m->ev_ready, st));
    CUDA_TRY(cudaStreamWaitEvent(m->xstream, m->ev_ready, 0));
    // the previous exchange's peer copies out of this send buffer are done
    for (int p = 0; p < R; ++p)
      if (p != r && m->host.send_counts[p]) CUDA_TRY(cudaStreamWaitEvent(m->xstream, g->m[p]->ev_xdone, 0));
    PROF(m, 5, m->xstream, launch_gather_pack(u[r], m->dm.dof_stride, m->d_send, m->po_send,
                                              m->d_sendbuf, m->xstream));
    CUDA_TRY(cudaGetLastError());
    CUDA_TRY(cudaEventRecord(g->ev_packed[r], m->xstream));
  }
  for (int p = 0; p < R; ++p) {
    dgr_mesh mp = g->m[p];
    DeviceGuard dg(mp->dev_id);
    for (int r = 0; r < R; ++r) {
      const int64_t n = mp->host.recv_counts[r];
      if (r == p || !n) continue;
      dgr_mesh mr = g->m[r];
      CUDA_TRY(cudaStreamWaitEvent(mp->xstream, g->ev_packed[r], 0));
      CUDA_TRY(cudaMemcpyPeerAsync(mp->d_recvbuf + NF * mp->po_recv.off[r], mp->dev_id,
                                   mr->d_sendbuf + NF * mr->po_send.off[p], mr->dev_id,
                                   size_t(NF) * n * sizeof(double), mp->xstream));
    }
    PROF(mp, 5, mp->xstream, launch_scatter_unpack(u[p], mp->dm.dof_stride, mp->host.n_owned_dof,
                                                   mp->d_recvbuf, mp->po_recv, mp->xstream));
    CUDA_TRY(cudaGetLastError());
    CUDA_TRY(cudaEventRecord(mp->ev_xdone, mp->xstream));
  }
  return DGR_OK;
}

static dgr_status group_check(dgr_group g, const void* const* a, const void* const* b) {
  if (!g || !a || !b) return fail(DGR_ERR_ARG, "null group argument");
  for (size_t r = 0; r < g->m.size(); ++r)   // (a null stream is the legacy default stream)
    if (!a[r]) return fail(DGR_ERR_ARG, "null state entry");
  return DGR_OK;
}

extern "C" {

dgr_status dgr_group_create(dgr_mesh* meshes, int n, dgr_group* out) {
  if (!meshes || !out || n < 1) return fail(DGR_ERR_ARG, "null argument or n < 1");
  *out = nullptr;
  for (int r = 0; r < n; ++r) {
    dgr_mesh m = meshes[r];
    if (!m || !m->device) return fail(DGR_ERR_ARG, "null or host-only mesh in the group");
    if (m->host.nranks != n || m->host.rank != r)
      return fail(DGR_ERR_ARG, "meshes[r] must be rank r of n ranks");
    if (m->comm || m->group) return fail(DGR_ERR_STATE, "mesh already has a communicator or group");
    if (m->host.oct.size() != meshes[0]->host.oct.size())
      return fail(DGR_ERR_ARG, "meshes of different octrees");
  }
  for (int p = 0; p < n; ++p)
    for (int r = 0; r < n; ++r)
      if (p != r && meshes[p]->host.recv_counts[r] != meshes[r]->host.send_counts[p])
        return fail(DGR_ERR_TREE, "send/receive counts of a rank pair disagree");
  std::unique_ptr<dgr_group_s> g(new dgr_group_s());
  g->m.assign(meshes, meshes + n);
  g->ev_packed.assign(size_t(n), nullptr);
  for (int r = 0; r < n; ++r) {
    DeviceGuard dg(meshes[r]->dev_id);
    CUDA_TRY(cudaEventCreateWithFlags(&g->ev_packed[r], cudaEventDisableTiming));
    // every rank's exchange stream and events exist before the first exchange
    // (rank r's pack waits on its peers' ev_xdone)
    if (dgr_status e = ensure_xstream(meshes[r])) return e;
    for (int p = 0; p < n; ++p)
      if (p != r && meshes[r]->dev_id != meshes[p]->dev_id) {
        int ok = 0;
        CUDA_TRY(cudaDeviceCanAccessPeer(&ok, meshes[r]->dev_id, meshes[p]->dev_id));
        if (ok) {
          cudaError_t e = cudaDeviceEnablePeerAccess(meshes[p]->dev_id, 0);
          if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
          else CUDA_TRY(e);
        }
      }
  }
  for (int r = 0; r < n; ++r) meshes[r]->group = g.get();
  *out = g.release();
  return DGR_OK;
}

dgr_status dgr_group_ghost_exchange(dgr_group g, double* const* u, void* const* streams) {
  dgr_status s = group_check(g, reinterpret_cast<const void* const*>(u), streams);
  if (s) return s;
  if ((s = group_exchange(g, u, streams))) return s;
  for (size_t r = 0; r < g->m.size(); ++r) {
    DeviceGuard dg(g->m[r]->dev_id);
    CUDA_TRY(cudaStreamWaitEvent(static_cast<cudaStream_t>(streams[r]), g->m[r]->ev_xdone, 0));
  }
  return DGR_OK;
}

dgr_status dgr_group_rk4_step(dgr_group g, double dt, double* const* u, const dgr_params* prm,
                              void* const* streams) {
  dgr_status s = group_check(g, reinterpret_cast<const void* const*>(u), streams);
  if (s) return s;
  const int R = int(g->m.size());
  for (dgr_mesh m : g->m) m->launches = 0;
  for (int k = 0; k < 4; ++k) {
    std::vector<double*> cur(R);
    for (int r = 0; r < R; ++r) cur[r] = k == 0 ? u[r] : g->m[r]->d_us;
    if ((s = group_exchange(g, cur.data(), streams))) return s;
    for (int r = 0; r < R; ++r) {
      dgr_mesh m = g->m[r];
      DeviceGuard dg(m->dev_id);
      if ((s = stage(m, k, dt, u[r], m->d_us, m->d_acc, u[r], prm,
                     static_cast<cudaStream_t>(streams[r]), true)))
        return s;
    }
  }
  return DGR_OK;
}

dgr_status dgr_group_destroy(dgr_group g) {
  delete g;
  return DGR_OK;
}

}  // extern "C"
