// Octant-to-patch ("unzip"), Alg. 2 (L249-283) / §IV-A (L235-306).
//
// Gather formulation, in two kernels:
//  * k_interp computes every *interpolation slot* once: the value of a coarser
//    element's degree-6 tensor Lagrange interpolant at a half-grid
//    point that a hanging node of a finer element (Alg. 2 lines 4-5) or a
//    finer neighbour's padding point needs.  Slots are deduplicated on the
//    host (one per distinct (coarse element, point); on C3 the padding points
//    alone need 3.6x fewer slots than points) and evaluated per element by
//    three 1-D sweeps over the bounding box of its slots, thinnest axis first;
//    the element's 343 nodal values are gathered from the state u and from
//    coarser slots (one launch per dependency depth: hanging chains, R14).
//  * k_unzip then assembles each 13^3 patch as a pure gather through the
//    mesh's gather map (copy / injection of DOFs or hanging-node slots,
//    interpolated points from their slots) with coalesced stores, and
//    extrapolates outside a non-periodic domain (reading R12).  The fused RHS
//    (rhs_kernel.cu) performs the same gather itself, into shared memory.
#include <cuda_runtime.h>

#include "device.cuh"

namespace dgr {

__constant__ double c_uW13[13 * 7];
__constant__ double c_uWEXT[3 * 7];

void upload_unzip_tables(const double* w13, const double* wext) {
  cudaMemcpyToSymbol(c_uW13, w13, sizeof(double) * 91);
  cudaMemcpyToSymbol(c_uWEXT, wext, sizeof(double) * 21);
}

namespace {
constexpr int UZ_WARPS = 8;                 // = fields per CTA
constexpr int UZ_THREADS = 32 * UZ_WARPS;
#ifndef DGR_IP_FG
#define DGR_IP_FG 4
#endif
constexpr int IP_FG = DGR_IP_FG;            // fields per k_interp CTA
#ifndef DGR_IP_THREADS
#define DGR_IP_THREADS 128   // (A/B: 0.493 -> 0.488 ms on C3; 512: 0.675)
#endif
constexpr int IP_THREADS = DGR_IP_THREADS;   // (experiment builds: -DDGR_IP_THREADS=...)
// sweep scratch per field: a face group's box is at most IP_N1 = 4 points thick
// along its first sweep axis (host-checked in api.cu), so T1 = 49 x n1 and
// T2 = 7 x n2 x n1 <= 7 x 13 x 4 (29 KB per 4-field CTA: 6 CTAs per SM)
constexpr int IP_N1 = 4;
constexpr int IP_T1 = 49 * IP_N1, IP_T2 = 7 * 13 * IP_N1;
constexpr int IP_FIELD = NPT + IP_T1 + IP_T2;   // scratch doubles per field

// q = floor(i / n) for 0 <= i < 2^16, 1 <= n <= 13 (float reciprocal, exact here)
__device__ __forceinline__ int fdiv(int i, float rn) { return int((float(i) + 0.5f) * rn); }
}  // namespace

// One CTA per (element, group of IP_FG fields): the element's nodal values are
// staged once, then for each face group of its slots, sweep 1 along the
// group's face normal a1 (its bounding box is <= 4 points thick along it) over
// all 7x7 node rows, sweep 2 along a2, then each slot's value along a3 (same 1-D operation per
// axis as the oracle's definition: sum_m l_m(t2/2) v_m, m = 0..6, or a copy at
// even t2).
__global__ void __launch_bounds__(IP_THREADS)
    k_interp(DevMesh m, const double* __restrict__ u, int nf, int64_t first) {
  extern __shared__ __align__(16) double dyn[];
  __shared__ double W[91];
  const int4 el = m.iel[first + blockIdx.x];
  const int f0 = blockIdx.y * IP_FG;
  const int tid = threadIdx.x;
  const int64_t ds = m.dof_stride, as = m.aux_stride;
  double* Es = dyn;                              // [IP_FG][NPT]
  double* T1 = Es + IP_FG * NPT;                 // [IP_FG][IP_T1]
  double* T2 = T1 + IP_FG * IP_T1;               // [IP_FG][IP_T2]
  for (int i = tid; i < 91; i += IP_THREADS) W[i] = c_uW13[i];
  {
    // all index loads, then all value loads in flight (two memory round trips)
    constexpr int NIT = (IP_FG * NPT + IP_THREADS - 1) / IP_THREADS;
    int32_t xs[NIT];
#pragma unroll
    for (int it = 0; it < NIT; ++it) {
      const int i = tid + it * IP_THREADS;
      const int g = i / NPT, n = i - g * NPT;
      xs[it] = (i < IP_FG * NPT && f0 + g < nf) ? __ldg(m.o2s + int64_t(el.x) * NPT + n) : -1;
    }
    double v[NIT];
#pragma unroll
    for (int it = 0; it < NIT; ++it) {
      const int i = tid + it * IP_THREADS;
      const int g = i / NPT;
      const int32_t x = xs[it];
      // (slots of coarser elements were written by an earlier launch: plain load)
      v[it] = x < 0 ? 0.0 : (x < ds ? __ldg(u + (f0 + g) * ds + x) : m.aux[(f0 + g) * as + (x - ds)]);
    }
#pragma unroll
    for (int it = 0; it < NIT; ++it) {
      const int i = tid + it * IP_THREADS;
      if (i < IP_FG * NPT) Es[i] = v[it];
    }
  }
  __syncthreads();
  for (int gi = 0; gi < el.z; ++gi) {
  const int4 gr = m.igrp[el.y + gi];
  const int a1 = (gr.z >> 24) & 3;   // the group's face normal (host-chosen, partition-invariant)
  const int a2 = a1 == 0 ? 1 : 0, a3 = a1 == 2 ? 1 : 2;
  // bounding box along a1 and a2 (4-bit fields: lo at 4a, hi at 12 + 4a)
  const int lo1 = (gr.z >> (4 * a1)) & 15, lo2 = (gr.z >> (4 * a2)) & 15;
  const int n1 = ((gr.z >> (12 + 4 * a1)) & 15) - lo1 + 1, n2 = ((gr.z >> (12 + 4 * a2)) & 15) - lo2 + 1;
  const int es1 = a1 == 0 ? 1 : (a1 == 1 ? 7 : 49);
  const int es2 = a2 == 0 ? 1 : (a2 == 1 ? 7 : 49);
  const int es3 = a3 == 0 ? 1 : (a3 == 1 ? 7 : 49);
  const float rn1 = 1.0f / float(n1), rn2 = 1.0f / float(n2);
  // this thread's slots of the group (k = tid + IP_THREADS i): their half-grid
  // points are loaded now, so the last sweep does not wait on global loads
  constexpr int IP_KMAX = (13 * 13 * IP_N1 + IP_THREADS - 1) / IP_THREADS;   // slots <= box volume
  uint32_t tk[IP_KMAX];
#pragma unroll
  for (int i = 0; i < IP_KMAX; ++i) {
    const int k = tid + IP_THREADS * i;
    tk[i] = k < gr.y ? __ldg(m.ipt + gr.x + k) : 0u;
  }
  // T1[g][r3][r2][i1] = sum_m W[lo1+i1][m] E_g[m, r2, r3]
  for (int idx = tid; idx < 49 * n1; idx += IP_THREADS) {
    const int r = fdiv(idx, rn1), i1 = idx - r * n1;   // r = r3 * 7 + r2
    const int r3 = r / 7, r2 = r - r3 * 7;
    const int row = r2 * es2 + r3 * es3;
    const int tt = lo1 + i1;
    double v[IP_FG];
    if (tt & 1) {
      const double* w = W + tt * 7;
#pragma unroll
      for (int g = 0; g < IP_FG; ++g) v[g] = 0.0;
#pragma unroll
      for (int q = 0; q < 7; ++q) {
        const double wq = w[q];
#pragma unroll
        for (int g = 0; g < IP_FG; ++g) v[g] = fma(wq, Es[g * NPT + row + q * es1], v[g]);
      }
    } else {
#pragma unroll
      for (int g = 0; g < IP_FG; ++g) v[g] = Es[g * NPT + row + (tt >> 1) * es1];
    }
#pragma unroll
    for (int g = 0; g < IP_FG; ++g) T1[g * IP_T1 + r * n1 + i1] = v[g];
  }
  __syncthreads();
  // T2[g][r3][i2][i1] = sum_m W[lo2+i2][m] T1[g][r3][m][i1]
  for (int idx = tid; idx < 7 * n2 * n1; idx += IP_THREADS) {
    const int q12 = fdiv(idx, rn1), i1 = idx - q12 * n1;
    const int r3 = fdiv(q12, rn2), i2 = q12 - r3 * n2;
    const int tt = lo2 + i2;
    const int col = r3 * 7 * n1 + i1;
    double v[IP_FG];
    if (tt & 1) {
      const double* w = W + tt * 7;
#pragma unroll
      for (int g = 0; g < IP_FG; ++g) v[g] = 0.0;
#pragma unroll
      for (int q = 0; q < 7; ++q) {
        const double wq = w[q];
#pragma unroll
        for (int g = 0; g < IP_FG; ++g) v[g] = fma(wq, T1[g * IP_T1 + col + q * n1], v[g]);
      }
    } else {
#pragma unroll
      for (int g = 0; g < IP_FG; ++g) v[g] = T1[g * IP_T1 + col + (tt >> 1) * n1];
    }
#pragma unroll
    for (int g = 0; g < IP_FG; ++g) T2[g * IP_T2 + (r3 * n2 + i2) * n1 + i1] = v[g];
  }
  __syncthreads();
  // slot value = sum_m W[t2_a3][m] T2[g][m][i2][i1]
  double* out = m.aux + gr.x;
#pragma unroll
  for (int ii = 0; ii < IP_KMAX; ++ii) {
    const int k = tid + IP_THREADS * ii;
    if (k < gr.y) {
    // (axis fields by shifts: a runtime-indexed local array would live in local memory)
    const int t = int(tk[ii]);
    const int i1 = ((t >> (4 * a1)) & 15) - lo1, i2 = ((t >> (4 * a2)) & 15) - lo2,
              tt = (t >> (4 * a3)) & 15;
    const int col = i2 * n1 + i1, st = n2 * n1;
    double v[IP_FG];
    if (tt & 1) {
      const double* w = W + tt * 7;
#pragma unroll
      for (int g = 0; g < IP_FG; ++g) v[g] = 0.0;
#pragma unroll
      for (int q = 0; q < 7; ++q) {
        const double wq = w[q];
#pragma unroll
        for (int g = 0; g < IP_FG; ++g) v[g] = fma(wq, T2[g * IP_T2 + col + q * st], v[g]);
      }
    } else {
#pragma unroll
      for (int g = 0; g < IP_FG; ++g) v[g] = T2[g * IP_T2 + col + (tt >> 1) * st];
    }
#pragma unroll
    for (int g = 0; g < IP_FG; ++g)
      if (f0 + g < nf) out[(f0 + g) * as + k] = v[g];
    }
  }
  __syncthreads();   // T1/T2 reused by the next group
  }  // face groups
}

void launch_interp(const DevMesh& m, const double* u, int nf, int64_t first, int64_t count,
                   cudaStream_t s) {
  if (count <= 0) return;
  const size_t dyn = size_t(IP_FG) * IP_FIELD * sizeof(double);
  static std::atomic<bool> done[MAX_DEVICES];
  if (first_on_device(done))
    cudaFuncSetAttribute(k_interp, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn));
  k_interp<<<dim3(unsigned(count), (nf + IP_FG - 1) / IP_FG), IP_THREADS, dyn, s>>>(m, u, nf,
                                                                                    first);
}

// One CTA per patch, ONE WARP PER FIELD (warp w builds fields w, w+8, w+16):
// copies with 8 loads in flight per lane and coalesced stores, then the
// outer-boundary extrapolation along x, y, z (boundary octants only) in three
// warp-synchronous passes over the patch just written.
#ifndef DGR_UZ_MINB
#define DGR_UZ_MINB 4   // (A/B, profiles/r2ab_*, r2ac_*: 14 loads in flight x 4 CTAs per SM: 2.51 -> 2.45 ms on C3)
#endif
#ifndef DGR_UZ_U
#define DGR_UZ_U 14
#endif
__global__ void __launch_bounds__(UZ_THREADS, DGR_UZ_MINB)
    k_unzip(DevMesh m, const double* __restrict__ u, double* __restrict__ patches, int nf) {
  __shared__ int32_t soff[NPATCH];
  __shared__ double WX[21];
  const int e = blockIdx.x;
  const int tid = threadIdx.x;
  const int lane = tid & 31, warp = tid >> 5;
  {
    const int32_t* gm = m.gmap + int64_t(e) * GM_PITCH;
    for (int p = tid; p < NPATCH; p += UZ_THREADS) soff[p] = __ldg(gm + p);   // -1: extrapolated
    for (int i = tid; i < 21; i += UZ_THREADS) WX[i] = c_uWEXT[i];
  }
  __syncthreads();

  const int64_t ds = m.dof_stride;
  for (int f = warp; f < nf; f += UZ_WARPS) {
  const double* uf = u + f * ds;
  const double* af = m.aux + f * m.aux_stride - ds;   // slot i - ds
  double* dst = patches + (int64_t(f) * m.n_owned + e) * PATCH_PITCH;

  // ---- gather: 16 loads in flight per lane; coalesced streaming (evict-first)
  // stores, so the 10-GB patch stream does not evict the element values and
  // slots the neighbouring patches still gather from L2
  constexpr int U = DGR_UZ_U;   // loads in flight per lane (experiment builds: -DDGR_UZ_U=...)
  for (int p0 = 0; p0 < NPATCH; p0 += 32 * U) {
    double v[U];
    int o[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int p = p0 + u * 32 + lane;
      o[u] = p < NPATCH ? soff[p] : -3;
      // (volatile asm keeps all U loads ahead of the stores; invalid points load
      // element value 0 and are not stored)
      const int x = max(o[u], 0);
      asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(v[u]) : "l"((x < ds ? uf : af) + x));
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (o[u] >= 0) __stcs(dst + p0 + u * 32 + lane, v[u]);
  }

  // ---- outer-boundary extrapolation along x, then y, then z (reading R12)
  const int4 oi = m.oct[e];
  if (!m.periodic) {
    const int64_t nside = int64_t(1) << m.D;
    const int64_t s = int64_t(1) << (m.D - oi.w);
    const bool out_lo[3] = {oi.x == 0, oi.y == 0, oi.z == 0};
    const bool out_hi[3] = {oi.x + s == nside, oi.y + s == nside, oi.z + s == nside};
    if (out_lo[0] || out_lo[1] || out_lo[2] || out_hi[0] || out_hi[1] || out_hi[2]) {
      for (int a = 0; a < 3; ++a) {
        __syncwarp();                                // previous writes visible to the warp
        const int sa = a == 0 ? 1 : (a == 1 ? 13 : 169);
        const int sb = a == 0 ? 13 : 1, sc = a == 2 ? 13 : 169;
        const int b_ax = a == 0 ? 1 : 0, c_ax = a == 2 ? 1 : 2;
        for (int side = 0; side < 2; ++side) {
          if (!(side == 0 ? out_lo[a] : out_hi[a])) continue;
          for (int idx = lane; idx < 3 * 169; idx += 32) {
            const int k3 = idx % 3, uv = idx / 3;
            const int cb = uv % 13, cc = uv / 13;
            if (b_ax > a && ((cb < 3 && out_lo[b_ax]) || (cb > 9 && out_hi[b_ax]))) continue;
            if (c_ax > a && ((cc < 3 && out_lo[c_ax]) || (cc > 9 && out_hi[c_ax]))) continue;
            const int ia = side == 0 ? k3 : 10 + k3;
            const int base = cb * sb + cc * sc;
            double acc = 0.0;
            if (side == 0) {
              const double* w = WX + (2 - ia) * 7;       // t = -(3 - ia)
#pragma unroll
              for (int mm = 0; mm < 7; ++mm)
                acc = fma(w[mm], __ldcg(dst + base + (3 + mm) * sa), acc);
            } else {
              const double* w = WX + (ia - 10) * 7;      // mirrored
#pragma unroll
              for (int mm = 0; mm < 7; ++mm)
                acc = fma(w[mm], __ldcg(dst + base + (9 - mm) * sa), acc);
            }
            dst[base + ia * sa] = acc;
          }
        }
      }
    }
  }
  }  // field loop
}

void launch_unzip(const DevMesh& m, const double* u, double* patches, int nf, cudaStream_t s) {
  if (m.n_owned <= 0) return;
  k_unzip<<<m.n_owned, UZ_THREADS, 0, s>>>(m, u, patches, nf);
}

}  // namespace dgr
