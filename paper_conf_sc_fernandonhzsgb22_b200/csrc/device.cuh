// Device-side data structures and kernel entry points of libdgr (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "host_mesh.hpp"

namespace dgr {

constexpr int NF = 24;            // BSSN fields
constexpr int PATCH_PITCH = 2208; // doubles per patch: 13^3 = 2197 padded to 128 B
constexpr int STAGE_DBL = 2200;   // smem stage buffer (bulk copy of 2200 doubles)
constexpr int GM_PITCH = 2200;    // int32 per octant in the fused-unzip gather map (16-B rows)

// Device view of a mesh (plain pointers; passed by value to kernels).
struct DevMesh {
  int32_t n_owned;      // owned octants
  int32_t n_local;      // owned + ghost octants
  int64_t dof_stride;
  int32_t n_owned_dof;
  int32_t D;
  int32_t periodic;
  double width;
  const int4* oct;          // [n_local] anchor x,y,z, level
  const int32_t* o2n;       // [n_local * 343] local DOF id or -1
  const uint8_t* pmap;      // [n_owned * 2197]
  const NbrEntry* nbr;      // [n_owned * NBR_MAX]
  const int32_t* zip;       // [n_owned_dof] local octant * 343 + node
  const int4* hang;         // rows: e_local, node, src_local, t2 packed (x | y<<8 | z<<16)
  // Patch gather: per field the source array SRC_f = E + f * e_stride holds
  // [element values of the n_local octants (n_local*343) | interpolation slots (n_interp)].
  // A slot is one distinct (coarse source element, half-grid point) pair that some
  // patch point interpolates from a coarser neighbour (deduplicated over all patches).
  // gmap[e][p] is the SRC_f index of patch point p of owned octant e, or -1 for a point
  // outside a non-periodic domain (extrapolated).
  int64_t e_stride;         // doubles per field of E (>= n_local*343 + n_interp)
  const int32_t* gmap;      // [n_owned * GM_PITCH]
  // interpolation work, one entry per coarse source element:
  //   {element, first slot, slot count, bbox lo (x|y<<4|z<<8) | hi << 12}
  const int4* iel;
  int32_t n_iel;
  const uint16_t* ipt;      // [n_interp] half-grid point of each slot, t2x | t2y<<4 | t2z<<8
};

// kernels.cu
void launch_elements(const DevMesh& m, const double* u, double* E, int nf, cudaStream_t s);
void launch_hanging(const DevMesh& m, const int4* rows, int64_t count, double* E, int nf,
                    cudaStream_t s);
void launch_unzip(const DevMesh& m, const double* E, double* patches, int nf, cudaStream_t s);
// interpolation slots (coarse-neighbour padding values) of E, from the element values
void launch_interp(const DevMesh& m, double* E, int nf, cudaStream_t s);
void launch_zip(const DevMesh& m, const double* rhs_oct, double* rhs, int nf, cudaStream_t s);
void launch_zip_rk4(const DevMesh& m, const double* rhs_oct, int stage, double dt,
                    const double* u_n, double* u_s, double* acc, double* u_out, cudaStream_t s);
void launch_dof_coords(const DevMesh& m, const int64_t* dof_node, double* xyz,
                       const double xmin[3], cudaStream_t s);
void launch_gather_pack(const double* u, int64_t stride, const int32_t* list, int64_t n,
                        double* buf, cudaStream_t s);
void launch_scatter_unpack(double* u, int64_t stride, int64_t offset, const double* buf,
                           int64_t n_total, cudaStream_t s);

void launch_dfma(int blocks, int iters, double* out, cudaStream_t s);

// rhs_kernel.cu
struct RhsParams {
  double ko_sigma, eta, lambda_f0, lambda_f1, chi_floor;
};
// Fused patch-to-octant + RK4 stage in the RHS epilogue (s < 0: write rhs_oct).
struct RkArgs {
  int s;
  double dt;
  const double* u_n;
  double* u_s;
  double* acc;
  double* u_out;
  const int32_t* own;   // [n_owned * 343]: owned DOF this point is the zip owner of, or -1
  int64_t stride;
};
// fused = false: read 13^3 patches ([24][n_owned][PATCH_PITCH], TMA bulk copies);
// fused = true: gather every patch from E through gmap (no patch buffer)
void launch_rhs(const DevMesh& m, const double* src, double* rhs_oct, const RhsParams& p,
                const RkArgs* rk, bool fused, cudaStream_t s);
size_t rhs_smem_bytes();
void upload_rhs_tables(const double* wext);

// constraints_kernel.cu
void launch_constraints(const DevMesh& m, const double* patches, double* c_oct,
                        const RhsParams& p, cudaStream_t s);

}  // namespace dgr
