// Unzip (octant-to-patch), element reconstruction, zip (patch-to-octant) and
// the fused zip + RK4 stage kernels (sm_100a, fp64).
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
__constant__ double c_W13[13 * 7];
__constant__ double c_WEXT[3 * 7];

void upload_tables(const double* w13, const double* wext) {
  cudaMemcpyToSymbol(c_W13, w13, sizeof(double) * 91);
  cudaMemcpyToSymbol(c_WEXT, wext, sizeof(double) * 21);
}

// I_c(t2) = sum_{ijk} W[t2x][i] W[t2y][j] W[t2z][k] E_c[i + 7j + 49k]; along an
// axis with even t2 the row is a unit vector: a single term.
__device__ __forceinline__ double interp_point(const double* __restrict__ Ec, int tx, int ty,
                                               int tz, const double* __restrict__ W) {
  const int nx = (tx & 1) ? 7 : 1, ny = (ty & 1) ? 7 : 1, nz = (tz & 1) ? 7 : 1;
  const int x0 = (tx & 1) ? 0 : (tx >> 1), y0 = (ty & 1) ? 0 : (ty >> 1),
            z0 = (tz & 1) ? 0 : (tz >> 1);
  double acc = 0.0;
  for (int c = 0; c < nz; ++c) {
    const double wz = (tz & 1) ? W[tz * 7 + c] : 1.0;
    double accy = 0.0;
    for (int b = 0; b < ny; ++b) {
      const double wy = (ty & 1) ? W[ty * 7 + b] : 1.0;
      const double* row = Ec + (x0 + 7 * (y0 + b) + 49 * (z0 + c));
      double accx = 0.0;
      for (int a = 0; a < nx; ++a) {
        const double wx = (tx & 1) ? W[tx * 7 + a] : 1.0;
        accx = fma(wx, __ldg(row + a), accx);
      }
      accy = fma(wy, accx, accy);
    }
    acc = fma(wz, accy, acc);
  }
  return acc;
}

// ---------------------------------------------------------- element gather
// E[f][e][n] = u[f][O2N[e][n]] for DOF nodes (Alg. 2 line 2); hanging nodes
// are filled level by level by k_hanging.
__global__ void k_elements(const double* __restrict__ u, int64_t stride,
                           const int32_t* __restrict__ o2n, int64_t nn, double* __restrict__ E) {
  const int f = blockIdx.y;
  const double* uf = u + f * stride;
  double* Ef = E + f * nn;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < nn;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int32_t id = __ldg(o2n + i);
    Ef[i] = id >= 0 ? __ldg(uf + id) : 0.0;
  }
}

void launch_elements(const DevMesh& m, const double* u, double* E, int nf, cudaStream_t s) {
  const int64_t nn = int64_t(m.n_local) * NPT;
  int blocks = int((nn + 255) / 256);
  if (blocks > 148 * 16) blocks = 148 * 16;
  k_elements<<<dim3(blocks, nf), 256, 0, s>>>(u, m.dof_stride, m.o2n, nn, E);
}

// --------------------------------------------------------- hanging points
// interp_hanging (Alg. 2 lines 4-5): E[e][node] = I_src(t2), rows of one level.
__global__ void k_hanging(const int4* __restrict__ rows, int64_t count, double* __restrict__ E,
                          int64_t nn) {
  __shared__ double W[91];
  for (int i = threadIdx.x; i < 91; i += blockDim.x) W[i] = c_W13[i];
  __syncthreads();
  const int f = blockIdx.y;
  double* Ef = E + f * nn;
  for (int64_t r = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; r < count;
       r += int64_t(gridDim.x) * blockDim.x) {
    const int4 row = rows[r];
    const int tx = row.w & 0xff, ty = (row.w >> 8) & 0xff, tz = (row.w >> 16) & 0xff;
    Ef[int64_t(row.x) * NPT + row.y] = interp_point(Ef + int64_t(row.z) * NPT, tx, ty, tz, W);
  }
}

void launch_hanging(const DevMesh& m, const int4* rows, int64_t count, double* E, int nf,
                    cudaStream_t s) {
  if (count <= 0) return;
  int blocks = int((count + 127) / 128);
  if (blocks > 148 * 16) blocks = 148 * 16;
  k_hanging<<<dim3(blocks, nf), 128, 0, s>>>(rows, count, E, int64_t(m.n_local) * NPT);
}

// ------------------------------------------------------------------ unzip
// One CTA per patch, fields in sequence.  Phase A: points sourced from the
// octant itself, a same-level or a finer neighbour are single loads (their
// half-grid coordinates are even); points sourced from a coarser neighbour c
// are produced by three 1D Lagrange sweeps over c's 7^3 nodes staged in shared
// memory, restricted to the bounding box of the points c sources (the
// tensor-product interpolation of P:L295).  Phase B: outer-boundary
// extrapolation (reading R12).  The finished 13^3 patch leaves shared memory
// with coalesced stores.
constexpr int UZ_THREADS = 256;
constexpr int UZ_FCHUNK = 4;   // fields per CTA: a wave of CTAs works on the same 4 fields (L2 reuse of E)

__global__ void __launch_bounds__(UZ_THREADS) k_unzip(DevMesh m, const double* __restrict__ E,
                                                      double* __restrict__ patches, int nf) {
  __shared__ __align__(16) double P[NPATCH + 3];
  __shared__ double Es[NPT + 1];
  __shared__ double T1[7 * 7 * 13];
  __shared__ double T2[7 * 13 * 13];
  __shared__ uint8_t pm[NPATCH + 11];
  __shared__ NbrEntry nb[NBR_MAX];
  __shared__ double W[91];
  __shared__ double WX[21];
  __shared__ int coarse[8];
  __shared__ int n_coarse;
  const int e = blockIdx.x;
  const int tid = threadIdx.x;
  for (int i = tid; i < NPATCH; i += UZ_THREADS) pm[i] = m.pmap[int64_t(e) * NPATCH + i];
  for (int i = tid; i < NBR_MAX; i += UZ_THREADS) nb[i] = m.nbr[int64_t(e) * NBR_MAX + i];
  for (int i = tid; i < 91; i += UZ_THREADS) W[i] = c_W13[i];
  for (int i = tid; i < 21; i += UZ_THREADS) WX[i] = c_WEXT[i];
  __syncthreads();
  if (tid == 0) {
    int nc = 0;
    for (int j = 0; j < NBR_MAX && nc < 8; ++j)
      if (nb[j].r == 1) coarse[nc++] = j;
    n_coarse = nc;
  }
  const int4 o = m.oct[e];
  const int64_t nside = int64_t(1) << m.D;
  const int64_t s = int64_t(1) << (m.D - o.w);
  const bool out_lo[3] = {!m.periodic && o.x == 0, !m.periodic && o.y == 0,
                          !m.periodic && o.z == 0};
  const bool out_hi[3] = {!m.periodic && o.x + s == nside, !m.periodic && o.y + s == nside,
                          !m.periodic && o.z + s == nside};
  const bool any_out = out_lo[0] || out_lo[1] || out_lo[2] || out_hi[0] || out_hi[1] || out_hi[2];
  __syncthreads();
  const int nc = n_coarse;
  const int64_t nn = int64_t(m.n_local) * NPT;
  const int f0 = blockIdx.y * UZ_FCHUNK, f1 = min(nf, f0 + UZ_FCHUNK);
  for (int f = f0; f < f1; ++f) {
    const double* Ef = E + f * nn;
    // ---- phase A.1: self / same level / finer: one load per point.  All of a
    // thread's source addresses are formed first so its ~9 loads are in flight
    // together (the kernel is load-latency bound otherwise).
    {
      constexpr int PER = (NPATCH + UZ_THREADS - 1) / UZ_THREADS;
      int64_t addr[PER];
#pragma unroll
      for (int q = 0; q < PER; ++q) {
        const int p = tid + q * UZ_THREADS;
        addr[q] = -1;
        if (p < NPATCH) {
          const int j = pm[p];
          const int ix = p % 13, iy = (p / 13) % 13, iz = p / 169;
          if (j == PM_SELF) {
            addr[q] = int64_t(e) * NPT + (ix - 3) + 7 * (iy - 3) + 49 * (iz - 3);
          } else if (j != PM_EXTRAP && nb[j].r != 1) {
            const NbrEntry& t = nb[j];
            const int tx = (t.o[0] + t.r * ix) >> 1, ty = (t.o[1] + t.r * iy) >> 1,
                      tz = (t.o[2] + t.r * iz) >> 1;
            addr[q] = int64_t(t.src) * NPT + tx + 7 * ty + 49 * tz;
          }
        }
      }
      double v[PER];
#pragma unroll
      for (int q = 0; q < PER; ++q) v[q] = addr[q] >= 0 ? __ldg(Ef + addr[q]) : 0.0;
#pragma unroll
      for (int q = 0; q < PER; ++q)
        if (addr[q] >= 0) P[tid + q * UZ_THREADS] = v[q];
    }
    // ---- phase A.2: coarser neighbours, separable sweeps x -> y -> z
    for (int ci = 0; ci < nc; ++ci) {
      const int j = coarse[ci];
      const NbrEntry t = nb[j];
      __syncthreads();   // previous users of Es / T1 / T2 are done
      const double* Ec = Ef + int64_t(t.src) * NPT;
      for (int i = tid; i < NPT; i += UZ_THREADS) Es[i] = __ldg(Ec + i);
      const int lx = t.lo[0], ly = t.lo[1], lz = t.lo[2];
      const int nx = t.hi[0] - lx + 1, ny = t.hi[1] - ly + 1, nz = t.hi[2] - lz + 1;
      __syncthreads();
      for (int idx = tid; idx < 49 * nx; idx += UZ_THREADS) {
        const int cyz = idx / nx, ix = idx % nx;        // cyz = cz * 7 + cy
        const int tx = t.o[0] + lx + ix;
        const double* row = Es + cyz * 7;
        double v;
        if (tx & 1) {
          const double* w = W + tx * 7;
          v = 0.0;
#pragma unroll
          for (int a = 0; a < 7; ++a) v = fma(w[a], row[a], v);
        } else {
          v = row[tx >> 1];
        }
        T1[cyz * 13 + ix] = v;
      }
      __syncthreads();
      for (int idx = tid; idx < 7 * ny * nx; idx += UZ_THREADS) {
        const int ix = idx % nx, iy = (idx / nx) % ny, cz = idx / (nx * ny);
        const int ty = t.o[1] + ly + iy;
        double v;
        if (ty & 1) {
          const double* w = W + ty * 7;
          v = 0.0;
#pragma unroll
          for (int b = 0; b < 7; ++b) v = fma(w[b], T1[(cz * 7 + b) * 13 + ix], v);
        } else {
          v = T1[(cz * 7 + (ty >> 1)) * 13 + ix];
        }
        T2[(cz * 13 + iy) * 13 + ix] = v;
      }
      __syncthreads();
      for (int idx = tid; idx < nz * ny * nx; idx += UZ_THREADS) {
        const int ix = idx % nx, iy = (idx / nx) % ny, iz = idx / (nx * ny);
        const int p = (lx + ix) + 13 * (ly + iy) + 169 * (lz + iz);
        if (pm[p] != j) continue;
        const int tz = t.o[2] + lz + iz;
        double v;
        if (tz & 1) {
          const double* w = W + tz * 7;
          v = 0.0;
#pragma unroll
          for (int c = 0; c < 7; ++c) v = fma(w[c], T2[(c * 13 + iy) * 13 + ix], v);
        } else {
          v = T2[((tz >> 1) * 13 + iy) * 13 + ix];
        }
        P[p] = v;
      }
    }
    if (any_out) {
      // Phase B (reading R12): degree-6 extrapolation along x, then y, then z,
      // for points outside along that axis and inside along all later axes.
      for (int a = 0; a < 3; ++a) {
        __syncthreads();
        for (int p = tid; p < NPATCH; p += UZ_THREADS) {
          const int idx[3] = {p % 13, (p / 13) % 13, p / 169};
          const int ia = idx[a];
          const bool outa = (ia < 3 && out_lo[a]) || (ia > 9 && out_hi[a]);
          if (!outa) continue;
          bool later_in = true;
          for (int b = a + 1; b < 3; ++b)
            if ((idx[b] < 3 && out_lo[b]) || (idx[b] > 9 && out_hi[b])) later_in = false;
          if (!later_in) continue;
          const int stride_a = a == 0 ? 1 : (a == 1 ? 13 : 169);
          const int base = p - ia * stride_a;
          double acc = 0.0;
          if (ia < 3) {
            const double* w = WX + (2 - ia) * 7;       // t = -(3 - ia)
            for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], P[base + (3 + mm) * stride_a], acc);
          } else {
            const double* w = WX + (ia - 10) * 7;      // mirrored
            for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], P[base + (9 - mm) * stride_a], acc);
          }
          P[p] = acc;
        }
      }
    }
    __syncthreads();
    double* dst = patches + (int64_t(f) * m.n_owned + e) * PATCH_PITCH;
    for (int p = tid; p < NPATCH; p += UZ_THREADS) __stcs(dst + p, P[p]);   // streaming: keep E in L2
    __syncthreads();
  }
}

void launch_unzip(const DevMesh& m, const double* E, double* patches, int nf, cudaStream_t s) {
  if (m.n_owned <= 0) return;
  k_unzip<<<dim3(m.n_owned, (nf + UZ_FCHUNK - 1) / UZ_FCHUNK), UZ_THREADS, 0, s>>>(m, E, patches, nf);
}

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
    if (S == 0) {
      const double un = u_n[i];
      acc[i] = un + (dt / 6.0) * k;
      u_s[i] = un + (dt / 2.0) * k;
    } else if (S == 1) {
      acc[i] += (dt / 3.0) * k;
      u_s[i] = u_n[i] + (dt / 2.0) * k;
    } else if (S == 2) {
      acc[i] += (dt / 3.0) * k;
      u_s[i] = u_n[i] + dt * k;
    } else {
      u_out[i] = acc[i] + (dt / 6.0) * k;
    }
  }
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

// ------------------------------------------------------- ghost pack/unpack
__global__ void k_pack(const double* __restrict__ u, int64_t stride,
                       const int32_t* __restrict__ list, int64_t n, double* __restrict__ buf) {
  // buf layout [f][n] per peer block is produced by the caller's offsets
  const int f = blockIdx.y;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x)
    buf[f * n + i] = u[f * stride + list[i]];
}

void launch_gather_pack(const double* u, int64_t stride, const int32_t* list, int64_t n,
                        double* buf, cudaStream_t s) {
  if (n <= 0) return;
  int blocks = int((n + 255) / 256);
  if (blocks > 148 * 4) blocks = 148 * 4;
  k_pack<<<dim3(blocks, NF), 256, 0, s>>>(u, stride, list, n, buf);
}

__global__ void k_unpack(double* __restrict__ u, int64_t stride, int64_t offset,
                         const double* __restrict__ buf, int64_t n) {
  const int f = blockIdx.y;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x)
    u[f * stride + offset + i] = buf[f * n + i];
}

void launch_scatter_unpack(double* u, int64_t stride, int64_t offset, const double* buf,
                           int64_t n_total, cudaStream_t s) {
  if (n_total <= 0) return;
  int blocks = int((n_total + 255) / 256);
  if (blocks > 148 * 4) blocks = 148 * 4;
  k_unpack<<<dim3(blocks, NF), 256, 0, s>>>(u, stride, offset, buf, n_total);
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
