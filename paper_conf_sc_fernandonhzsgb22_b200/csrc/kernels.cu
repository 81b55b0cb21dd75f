// Zip (patch-to-octant), the fused zip + RK4 stage kernels, DOF coordinates,
// ghost pack/unpack and the fp64 microbenchmark (sm_100a, fp64).  Octant-to-
// patch (unzip, hanging nodes, interpolation): unzip_kernel.cu.
//
// PAPER.md Alg. 2 (L249-283) / §IV-A (L235-306): octant-to-patch fills the
// (r+2k)^3 = 13^3 padded patch of every octant by copy (same level), injection
// (neighbour finer) or interpolation (neighbour coarser).  The paper scatters
// from each octant into its neighbours' patches (grid (|E|, dof), block (r,r));
// on B200 we GATHER per patch instead: one CTA owns one patch, assembles it in
// shared memory and writes it with full, coalesced 128-B lines (the patch
// writes are ~90% of the kernel's bytes).
#include <cuda_runtime.h>

#include "device.cuh"

namespace dgr {

// Lagrange rows: [t2][m] = l_m(t2/2), degree 6 on nodes 0..6;
// extrapolation rows [t][m] = l_m(-(t+1)).  Filled by the host (api.cu).
void upload_unzip_tables(const double* w13, const double* wext);  // unzip_kernel.cu

void upload_tables(const double* w13, const double* wext) { upload_unzip_tables(w13, wext); }

// (octant-to-patch: unzip_kernel.cu)

// -------------------------------------------------------------------- zip
// Patch-to-octant: each owned DOF takes its zip owner's value.
__global__ void k_zip(const int32_t* __restrict__ zip, int32_t n, int64_t no343,
                      const double* __restrict__ rhs_oct, double* __restrict__ rhs,
                      int64_t stride) {
  const int f = blockIdx.y;
  for (int d = blockIdx.x * blockDim.x + threadIdx.x; d < n; d += gridDim.x * blockDim.x)
    rhs[f * stride + d] = __ldg(rhs_oct + f * no343 + __ldg(zip + d));
}

void launch_zip(const DevMesh& m, const double* rhs_oct, double* rhs, int nf, cudaStream_t s) {
  if (m.n_owned_dof <= 0) return;
  int blocks = (m.n_owned_dof + 255) / 256;
  if (blocks > 148 * 8) blocks = 148 * 8;
  k_zip<<<dim3(blocks, nf), 256, 0, s>>>(m.zip, m.n_owned_dof, int64_t(m.n_owned) * NPT, rhs_oct,
                                         rhs, m.dof_stride);
}

// Zip fused with the RK4 stage update (Alg. 1 lines 9-10; reading R11):
//   s=0: acc = u_n + dt/6 k; u_s = u_n + dt/2 k     s=1: acc += dt/3 k; u_s = u_n + dt/2 k
//   s=2: acc += dt/3 k;      u_s = u_n + dt k       s=3: u_out = acc + dt/6 k
template <int S>
__global__ void k_zip_rk4(const int32_t* __restrict__ zip, int32_t n, int64_t no343,
                          const double* __restrict__ rhs_oct, int64_t stride, double dt,
                          const double* __restrict__ u_n, double* __restrict__ u_s,
                          double* __restrict__ acc, double* __restrict__ u_out) {
  const int f = blockIdx.y;
  for (int d = blockIdx.x * blockDim.x + threadIdx.x; d < n; d += gridDim.x * blockDim.x) {
    const int64_t i = f * stride + d;
    const double k = __ldg(rhs_oct + f * no343 + __ldg(zip + d));
    rk4_update<S>(i, k, dt, u_n, u_s, acc, u_out);
  }
}

// The same update from an RHS already in DOF order (written by k_rhs's zip-
// by-store epilogue): every array is streamed, no zip gather.
template <int S>
__global__ void k_rk4(int32_t n, int64_t stride, double dt, const double* __restrict__ rhs,
                      const double* __restrict__ u_n, double* __restrict__ u_s,
                      double* __restrict__ acc, double* __restrict__ u_out) {
  const int f = blockIdx.y;
  for (int d = blockIdx.x * blockDim.x + threadIdx.x; d < n; d += gridDim.x * blockDim.x) {
    const int64_t i = f * stride + d;
    const double k = __ldcs(rhs + i);
    rk4_update<S>(i, k, dt, u_n, u_s, acc, u_out);
  }
}

void launch_rk4(const DevMesh& m, const double* rhs, int stage, double dt, const double* u_n,
                double* u_s, double* acc, double* u_out, cudaStream_t s) {
  if (m.n_owned_dof <= 0) return;
  int blocks = (m.n_owned_dof + 255) / 256;
  if (blocks > 148 * 8) blocks = 148 * 8;
  const dim3 g(blocks, NF);
  const int32_t n = m.n_owned_dof;
  switch (stage) {
    case 0: k_rk4<0><<<g, 256, 0, s>>>(n, m.dof_stride, dt, rhs, u_n, u_s, acc, u_out); break;
    case 1: k_rk4<1><<<g, 256, 0, s>>>(n, m.dof_stride, dt, rhs, u_n, u_s, acc, u_out); break;
    case 2: k_rk4<2><<<g, 256, 0, s>>>(n, m.dof_stride, dt, rhs, u_n, u_s, acc, u_out); break;
    default: k_rk4<3><<<g, 256, 0, s>>>(n, m.dof_stride, dt, rhs, u_n, u_s, acc, u_out); break;
  }
}

// ------------------------------------------------- constraint norms (a7)
// Sum of squares and max |.| of each of nq rows of c over d < n, in a fixed
// order (deterministic): per-block partials, then one block per row.
constexpr int CN_THREADS = 256;
__global__ void k_cnorm_partial(const double* __restrict__ c, int64_t stride, int64_t n,
                                double* __restrict__ part /*[nq][2][gridDim.x]*/) {
  const int q = blockIdx.y;
  double ss = 0.0, mx = 0.0;
  for (int64_t d = blockIdx.x * int64_t(CN_THREADS) + threadIdx.x; d < n;
       d += int64_t(gridDim.x) * CN_THREADS) {
    const double v = c[q * stride + d];
    ss = fma(v, v, ss);
    mx = fmax(mx, fabs(v));
  }
  __shared__ double s_ss[CN_THREADS], s_mx[CN_THREADS];
  s_ss[threadIdx.x] = ss;
  s_mx[threadIdx.x] = mx;
  __syncthreads();
  for (int w = CN_THREADS / 2; w > 0; w >>= 1) {
    if (int(threadIdx.x) < w) {
      s_ss[threadIdx.x] += s_ss[threadIdx.x + w];
      s_mx[threadIdx.x] = fmax(s_mx[threadIdx.x], s_mx[threadIdx.x + w]);
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    part[(2 * q) * gridDim.x + blockIdx.x] = s_ss[0];
    part[(2 * q + 1) * gridDim.x + blockIdx.x] = s_mx[0];
  }
}
__global__ void k_cnorm_final(const double* __restrict__ part, int nblk, double* __restrict__ out) {
  const int q = blockIdx.x;
  if (threadIdx.x == 0) {
    double ss = 0.0, mx = 0.0;
    for (int b = 0; b < nblk; ++b) {
      ss += part[(2 * q) * nblk + b];
      mx = fmax(mx, part[(2 * q + 1) * nblk + b]);
    }
    out[2 * q] = ss;
    out[2 * q + 1] = mx;
  }
}
void launch_cnorms(const double* c, int64_t stride, int64_t n, int nq, double* part, double* out,
                   cudaStream_t s) {
  k_cnorm_partial<<<dim3(CN_BLOCKS, nq), CN_THREADS, 0, s>>>(c, stride, n, part);
  k_cnorm_final<<<nq, 32, 0, s>>>(part, CN_BLOCKS, out);
}

void launch_zip_rk4(const DevMesh& m, const double* rhs_oct, int stage, double dt,
                    const double* u_n, double* u_s, double* acc, double* u_out, cudaStream_t s) {
  if (m.n_owned_dof <= 0) return;
  int blocks = (m.n_owned_dof + 255) / 256;
  if (blocks > 148 * 8) blocks = 148 * 8;
  const dim3 g(blocks, NF);
  const int64_t no343 = int64_t(m.n_owned) * NPT;
  switch (stage) {
    case 0: k_zip_rk4<0><<<g, 256, 0, s>>>(m.zip, m.n_owned_dof, no343, rhs_oct, m.dof_stride, dt, u_n, u_s, acc, u_out); break;
    case 1: k_zip_rk4<1><<<g, 256, 0, s>>>(m.zip, m.n_owned_dof, no343, rhs_oct, m.dof_stride, dt, u_n, u_s, acc, u_out); break;
    case 2: k_zip_rk4<2><<<g, 256, 0, s>>>(m.zip, m.n_owned_dof, no343, rhs_oct, m.dof_stride, dt, u_n, u_s, acc, u_out); break;
    default: k_zip_rk4<3><<<g, 256, 0, s>>>(m.zip, m.n_owned_dof, no343, rhs_oct, m.dof_stride, dt, u_n, u_s, acc, u_out); break;
  }
}

// ----------------------------------------------------------- coordinates
__global__ void k_dof_coords(const int64_t* __restrict__ node, int64_t n, int64_t stride,
                             double* __restrict__ xyz, double x0, double y0, double z0,
                             double unit) {
  for (int64_t d = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; d < n;
       d += int64_t(gridDim.x) * blockDim.x) {
    // explicit rounding (no FMA contraction): xmin + X * unit, as on the host
    xyz[d] = __dadd_rn(x0, __dmul_rn(double(node[3 * d + 0]), unit));
    xyz[stride + d] = __dadd_rn(y0, __dmul_rn(double(node[3 * d + 1]), unit));
    xyz[2 * stride + d] = __dadd_rn(z0, __dmul_rn(double(node[3 * d + 2]), unit));
  }
}

void launch_dof_coords(const DevMesh& m, const int64_t* dof_node, double* xyz,
                       const double xmin[3], cudaStream_t s) {
  const int64_t n = m.dof_stride;
  int blocks = int((n + 255) / 256);
  if (blocks > 148 * 8) blocks = 148 * 8;
  const double unit = m.width / double(6 * (int64_t(1) << m.D));
  k_dof_coords<<<blocks, 256, 0, s>>>(dof_node, n, m.dof_stride, xyz, xmin[0], xmin[1], xmin[2],
                                      unit);
}

// ------------------------------------------------------- per-device setup
bool first_on_device(std::atomic<bool>* flags) {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= MAX_DEVICES) return false;
  return !flags[dev].exchange(true);
}

int sm_count() {
  static std::atomic<int> cache[MAX_DEVICES];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= MAX_DEVICES) return 148;
  int n = cache[dev].load();
  if (!n) {
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
    cache[dev].store(n);
  }
  return n;
}

// ------------------------------------------------------- ghost pack/unpack
// Peer-major message layout (one contiguous message per peer):
// the n_p entries for peer p occupy buf[NF * off[p], NF * off[p + 1]) as a
// [NF][n_p] block, off = prefix sums of the per-peer counts (nranks + 1 entries,
// nranks <= MAX_RANKS).  Entry i belongs to the peer p with off[p] <= i < off[p+1].
__device__ __forceinline__ int peer_of(const int64_t* off, int np, int64_t i) {
  int p = 0;
  while (p + 1 < np && off[p + 1] <= i) ++p;
  return p;
}

__global__ void k_pack(const double* __restrict__ u, int64_t stride,
                       const int32_t* __restrict__ list, PeerOffsets po, double* __restrict__ buf) {
  const int f = blockIdx.y;
  const int64_t n = po.off[po.np];
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int p = peer_of(po.off, po.np, i);
    const int64_t o = po.off[p], np_ = po.off[p + 1] - o;
    buf[NF * o + f * np_ + (i - o)] = u[f * stride + list[i]];
  }
}

void launch_gather_pack(const double* u, int64_t stride, const int32_t* list, const PeerOffsets& po,
                        double* buf, cudaStream_t s) {
  const int64_t n = po.off[po.np];
  if (n <= 0) return;
  int blocks = int((n + 255) / 256);
  if (blocks > 148 * 4) blocks = 148 * 4;
  k_pack<<<dim3(blocks, NF), 256, 0, s>>>(u, stride, list, po, buf);
}

// ghost slice of u (peer-major: DOFs received from peer p at n_owned + off[p] ..)
// from the peer-major receive buffer
__global__ void k_unpack(double* __restrict__ u, int64_t stride, int64_t n_owned,
                         const double* __restrict__ buf, PeerOffsets po) {
  const int f = blockIdx.y;
  const int64_t n = po.off[po.np];
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int p = peer_of(po.off, po.np, i);
    const int64_t o = po.off[p], np_ = po.off[p + 1] - o;
    u[f * stride + n_owned + i] = buf[NF * o + f * np_ + (i - o)];
  }
}

void launch_scatter_unpack(double* u, int64_t stride, int64_t n_owned, const double* buf,
                           const PeerOffsets& po, cudaStream_t s) {
  const int64_t n = po.off[po.np];
  if (n <= 0) return;
  int blocks = int((n + 255) / 256);
  if (blocks > 148 * 4) blocks = 148 * 4;
  k_unpack<<<dim3(blocks, NF), 256, 0, s>>>(u, stride, n_owned, buf, po);
}

// ------------------------------------------------------ fp64 microbenchmark
__global__ void __launch_bounds__(256) k_dfma(int iters, double* out) {
  double a[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) a[k] = 1.0 + 1e-3 * (threadIdx.x + k);
  const double b = 0.9999999, c = 1e-7;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = fma(a[k], b, c);
  }
  double sum = 0.0;
#pragma unroll
  for (int k = 0; k < 8; ++k) sum += a[k];
  if (sum == 1234.5678) out[0] = sum;   // keeps the chains alive
}

void launch_dfma(int blocks, int iters, double* out, cudaStream_t s) {
  k_dfma<<<blocks, 256, 0, s>>>(iters, out);
}

}  // namespace dgr
