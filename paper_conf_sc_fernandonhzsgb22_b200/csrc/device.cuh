// Device-side data structures and kernel entry points of libdgr (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "host_mesh.hpp"

namespace dgr {

// Per-device one-time setup (kernel attributes are per device context): true
// the first time it is called for the current device with this flag array;
// thread-safe (a static bool / SM count cached from the first
// device broke meshes created on a second GPU in the same process).
constexpr int MAX_DEVICES = 64;
bool first_on_device(std::atomic<bool>* flags);
int sm_count();

constexpr int NF = 24;            // BSSN fields
constexpr int PATCH_PITCH = 2208; // doubles per patch: 13^3 = 2197 padded to 128 B
constexpr int STAGE_DBL = 2200;   // smem stage buffer (bulk copy of 2200 doubles)
constexpr int GM_PITCH = 2200;    // int32 per octant in the fused-unzip gather map (16-B rows)
// sorted gather rows (gmap_s): the first G_CROSS entries are the points a
// first-derivative stencil reads, the first G_SLABS those any stencil or the
// D1 pass reads (the 216 corner points come last and are never read)
constexpr int G_CROSS = 343 + 6 * 3 * 49;          // 1225
constexpr int G_SLABS = 2197 - 8 * 27;             // 1981

// Device view of a mesh (plain pointers; passed by value to kernels).
struct DevMesh {
  int32_t n_owned;      // owned octants
  int32_t n_local;      // owned + ghost octants
  int64_t dof_stride;
  int32_t n_owned_dof;
  int32_t D;
  int32_t periodic;
  double width;
  double xmin[3];           // physical coordinates of the domain corner
  const int4* oct;          // [n_local] anchor x,y,z, level
  const int32_t* o2n;       // [n_local * 343] local DOF id or -1
  const uint8_t* pmap;      // [n_owned * 2197]
  const NbrEntry* nbr;      // [n_owned * NBR_MAX]
  const int32_t* zip;       // [n_owned_dof] local octant * 343 + node
  const int32_t* own;       // [n_owned * 343] owned DOF whose zip owner is (e, p), or -1
  // Gather maps.  Index space of every value a patch needs:
  // i < dof_stride -> u[f * dof_stride + i] (a DOF of the state), else
  // aux[f * aux_stride + i - dof_stride] (an interpolation slot: one distinct
  // (coarse element, half-grid point) needed by a hanging node or by a padding
  // point sourced by a coarser neighbour, filled by k_interp).
  double* aux;              // [24][aux_stride]
  int64_t aux_stride;
  const int32_t* o2s;       // [n_local * 343] element node -> index
  // gmap[e][p]: index of patch point p of owned octant e, -1 outside a
  // non-periodic domain (extrapolated)
  const int32_t* gmap;      // [n_owned * GM_PITCH]
  // the fused kernels' gather: gmap entries sorted by source index (gmap_s)
  // and the patch point each one fills (gdst)
  const int32_t* gmap_s;
  const int16_t* gdst;
  // RHS octant order: interior octants (no ghost-dependent gather source)
  // first, then the boundary octants (api.cu, overlap of the ghost exchange)
  const int32_t* olist;     // [n_owned]
  // interpolation work: one entry per element with slots (sorted by dependency
  // depth) {element, first group, group count, 0}, and per face group of its
  // slots {first slot, slot count, bbox lo (x|y<<4|z<<8) | hi << 12 | first
  // sweep axis << 24, 0}
  const int4* iel;
  const int4* igrp;
  int32_t n_iel;
  const uint16_t* ipt;      // [n_interp] half-grid point of each slot, t2x | t2y<<4 | t2z<<8
};

// unzip_kernel.cu
void launch_unzip(const DevMesh& m, const double* u, double* patches, int nf, cudaStream_t s);
// interpolation slots of m.iel[first .. first + count) (one dependency depth)
void launch_interp(const DevMesh& m, const double* u, int nf, int64_t first, int64_t count,
                   cudaStream_t s);
// kernels.cu
void launch_zip(const DevMesh& m, const double* rhs_oct, double* rhs, int nf, cudaStream_t s);
// sums of squares and max |.| of rows q < nq of c over d < n -> out[2q], out[2q+1]
// (device; part: [nq][2][CN_BLOCKS] scratch)
constexpr int CN_BLOCKS = 296;
void launch_cnorms(const double* c, int64_t stride, int64_t n, int nq, double* part, double* out,
                   cudaStream_t s);
void launch_zip_rk4(const DevMesh& m, const double* rhs_oct, int stage, double dt,
                    const double* u_n, double* u_s, double* acc, double* u_out, cudaStream_t s);
// RK4 stage update from an already zipped RHS rhs[24][dof_stride] (streaming)
void launch_rk4(const DevMesh& m, const double* rhs, int stage, double dt, const double* u_n,
                double* u_s, double* acc, double* u_out, cudaStream_t s);
void launch_dof_coords(const DevMesh& m, const int64_t* dof_node, double* xyz,
                       const double xmin[3], cudaStream_t s);
// per-peer prefix offsets of a peer-major message buffer (passed by value)
constexpr int MAX_RANKS = 64;
struct PeerOffsets {
  int np;                       // number of peers (= nranks)
  int64_t off[MAX_RANKS + 1];   // off[p] = entries before peer p's block
};
// buf (peer-major, one [NF][n_p] block per peer p) <- u[f][list[i]]
void launch_gather_pack(const double* u, int64_t stride, const int32_t* list, const PeerOffsets& po,
                        double* buf, cudaStream_t s);
// u[f][n_owned + i] <- peer-major receive buffer
void launch_scatter_unpack(double* u, int64_t stride, int64_t n_owned, const double* buf,
                           const PeerOffsets& po, cudaStream_t s);

void launch_dfma(int blocks, int iters, double* out, cudaStream_t s);

// The RK4 stage update of element i from its RHS k (reading R11, classic
// tableau), with explicit fma so k_rk4, k_zip_rk4 and the fused k_rhs epilogue
// round alike:  s=0: acc = u_n + dt/6 k, u_s = u_n + dt/2 k;  s=1: acc += dt/3 k,
// u_s = u_n + dt/2 k;  s=2: acc += dt/3 k, u_s = u_n + dt k;  s=3: u_out = acc + dt/6 k
template <int S>
__device__ __forceinline__ void rk4_update(int64_t i, double k, double dt, const double* u_n,
                                           double* u_s, double* acc, double* u_out) {
  if (S == 0) {
    const double un = u_n[i];
    acc[i] = __fma_rn(dt / 6.0, k, un);
    u_s[i] = __fma_rn(dt / 2.0, k, un);
  } else if (S == 1) {
    acc[i] = __fma_rn(dt / 3.0, k, acc[i]);
    u_s[i] = __fma_rn(dt / 2.0, k, u_n[i]);
  } else if (S == 2) {
    acc[i] = __fma_rn(dt / 3.0, k, acc[i]);
    u_s[i] = __fma_rn(dt, k, u_n[i]);
  } else {
    u_out[i] = __fma_rn(dt / 6.0, k, acc[i]);
  }
}

// rhs_kernel.cu
struct RhsParams {
  double ko_sigma, eta, lambda_f0, lambda_f1, chi_floor;
  int sommerfeld;   // radiative outer boundary (reading R29)
  int upwind;       // lopsided advective derivatives (reading R9u)
  // RK4 stage update fused into the zip-by-store epilogue (rk_stage >= 0,
  // reading R11, the arithmetic of k_rk4): each zip owner updates its DOF's
  // acc / u_s (stage 0..2) or u_out (stage 3) instead of storing the RHS
  int rk_stage = -1;
  double rk_dt = 0.0;
  const double* rk_un = nullptr;
  double* rk_acc = nullptr;
  double* rk_us = nullptr;
  double* rk_out = nullptr;
};
// fused = false: read 13^3 patches ([24][n_owned][PATCH_PITCH], TMA bulk copies);
// fused = true: `src` is the state u; every patch is gathered from u and the
// slots through gmap (no patch buffer)
// RHS of the owned octants m.olist[first, first + count); at most
// n_SM - leave_sm persistent CTAs
// pre != nullptr (fused, no Sommerfeld): the gt_ij stages run in the metric
// pre-pass k_gt_pre (pre: [30][n_owned][343] scratch), then k_rhs on the rest
// rhs_dof != nullptr (fused, no Sommerfeld): the zip is done by the store — each
// point writes its 24 values to rhs_dof[f * dof_stride + d] iff it is the zip
// owner of DOF d (m.own), and rhs_oct is not written
void launch_rhs(const DevMesh& m, const double* src, double* rhs_oct, const RhsParams& p,
                bool fused, int64_t first, int64_t count, int leave_sm, cudaStream_t s,
                double* pre = nullptr, double* rhs_dof = nullptr);
size_t rhs_smem_bytes();
int pre_rows();   // metric pre-pass values per interior point
void upload_rhs_tables(const double* wext);

// gen/rhs_alg.cu (generated by codegen/gen.py): the algebraic part A of the RHS
// in the paper's code-generation styles (Table II), in[234][ld] -> out[24][ld];
// variant 0 sympygr_cse, 1 binary_reduce, 2 staged_cse; occ = 1: the
// occupancy-constrained build (256 threads x 4 CTAs per SM, <= 64 registers)
struct AlgParams {
  double eta, lambda_f0, lambda_f1, chi_floor;
};
void launch_rhs_alg(int variant, int occ, const double* in, double* out, int64_t n, int64_t ld,
                    const AlgParams& p, cudaStream_t s);
// rhs_inputs.cu: the 234 inputs of A per interior point from the patch buffer
void launch_rhs_inputs(const DevMesh& m, const double* patches, double* in, int64_t ld,
                       double ko_sigma, cudaStream_t s);

// regrid.cu (readings R30-R32): wavelet indicator per owned octant from the
// patch buffer (fields in `mask`), and the intergrid transfer of the new
// mesh's DOFs from the old mesh's element interpolants
void upload_regrid_tables(const double* w13);
void launch_wavelet(const DevMesh& m, const double* patches, uint32_t mask, double* w,
                    cudaStream_t s);
void launch_transfer(const DevMesh& old, const double* u_old, const int4* map, int64_t n,
                     double* u_new, int64_t new_stride, cudaStream_t s);

// gen/psi4.cu (generated) + psi4.cu: gravitational-wave extraction (R33-R36)
void launch_psi4(const double* in, const double* xyz, double* out, int64_t n, int64_t ld,
                 const AlgParams& p, cudaStream_t s);
void launch_octant_xyz(const DevMesh& m, const double c[3], double* xyz, int64_t ld,
                       cudaStream_t s);
void launch_sphere_interp(const double* psi, int64_t ld, const int32_t* oct, const double* t,
                          int64_t n, double* out, cudaStream_t s);

// constraints_kernel.cu
void launch_constraints(const DevMesh& m, const double* patches, double* c_oct,
                        const RhsParams& p, cudaStream_t s);

}  // namespace dgr
