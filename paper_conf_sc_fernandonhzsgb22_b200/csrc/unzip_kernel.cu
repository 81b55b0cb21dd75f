// Octant-to-patch ("unzip"), Alg. 2 (L249-283) / §IV-A (L235-306).
//
// Gather formulation.  One CTA per (patch, chunk of 8 fields)
// and ONE WARP PER FIELD: after a CTA-wide setup that resolves every patch
// point's source once (shared by the 8 warps), each warp assembles its field's
// 13^3 patch with no further CTA barriers:
//  * copy points (self / same-level / finer neighbour: even half-grid
//    coordinates) -> one load of a reconstructed nodal value, 8 loads in
//    flight per lane, coalesced stores straight to the patch buffer;
//  * points sourced by a coarser neighbour -> its 7^3 nodes staged in the
//    warp's shared scratch, an x-sweep of 1-D degree-6 Lagrange rows over the
//    bounding box of those points, then y/z rows per point (tensor-product
//    interpolation);
//  * outer-boundary extrapolation (reading R12) in three warp-synchronous
//    passes over the patch just written (boundary octants only).
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
constexpr int BOXMAX = 10;                  // coarse-source box: edges <= 10, thinnest <= 4
constexpr int T1N = 49 * 4;                 // (both host-checked)
constexpr int T2N = 7 * 4 * BOXMAX;
constexpr int WSCR = NPT + 1 + T1N + T2N;   // per-warp scratch (doubles)

// q = floor(i / n) for 0 <= i < 2^16, 1 <= n <= 13 (float reciprocal, exact here)
__device__ __forceinline__ int fdiv(int i, float rn) { return int((float(i) + 0.5f) * rn); }
}  // namespace

__global__ void __launch_bounds__(UZ_THREADS, 3)
    k_unzip(DevMesh m, const double* __restrict__ E, double* __restrict__ patches, int nf) {
  __shared__ __align__(16) uint8_t pm[PMAP_PITCH];
  __shared__ int32_t soff[NPATCH];
  __shared__ NbrEntry nb[NBR_MAX];
  __shared__ double W[91];
  __shared__ double WX[21];
  extern __shared__ __align__(16) double dyn[];   // per-warp scratch: Es, T1, T2
  __shared__ int coarse[8];
  __shared__ int n_coarse;
  const int e = blockIdx.x;
  const int tid = threadIdx.x;
  const int lane = tid & 31, warp = tid >> 5;
  {
    const uint4* src = reinterpret_cast<const uint4*>(m.pmap + int64_t(e) * PMAP_PITCH);
    uint4* dst = reinterpret_cast<uint4*>(pm);
    for (int i = tid; i < PMAP_PITCH / 16; i += UZ_THREADS) dst[i] = __ldg(src + i);
    const int* nsrc = reinterpret_cast<const int*>(m.nbr + int64_t(e) * NBR_MAX);
    int* ndst = reinterpret_cast<int*>(nb);
    for (int i = tid; i < NBR_MAX * int(sizeof(NbrEntry)) / 4; i += UZ_THREADS)
      ndst[i] = __ldg(nsrc + i);
    for (int i = tid; i < 91; i += UZ_THREADS) W[i] = c_uW13[i];
    for (int i = tid; i < 21; i += UZ_THREADS) WX[i] = c_uWEXT[i];
  }
  __syncthreads();
  // resolve every point's source once: element-buffer offset, -1 coarse, -2 extrapolated
  for (int p = tid; p < NPATCH; p += UZ_THREADS) {
    const int j = pm[p];
    const int ix = p % 13, iy = (p / 13) % 13, iz = p / 169;
    int off = -2;
    if (j == PM_SELF) {
      off = e * NPT + (ix - 3) + 7 * (iy - 3) + 49 * (iz - 3);
    } else if (j != PM_EXTRAP) {
      const NbrEntry& t = nb[j];
      if (t.r == 1) {
        off = -1;
      } else {
        const int tx = (t.o[0] + t.r * ix) >> 1, ty = (t.o[1] + t.r * iy) >> 1,
                  tz = (t.o[2] + t.r * iz) >> 1;
        off = t.src * NPT + tx + 7 * ty + 49 * tz;
      }
    }
    soff[p] = off;
  }
  if (tid == 0) {
    int nc = 0;
    for (int j = 0; j < NBR_MAX && nc < 8; ++j)
      if (nb[j].r == 1) coarse[nc++] = j;
    n_coarse = nc;
  }
  __syncthreads();

  // warp w builds fields w, w + 8, w + 16 (the setup above is done once per octant)
  const int64_t nn = int64_t(m.n_local) * NPT;
  for (int f = warp; f < nf; f += UZ_WARPS) {
  const double* Ef = E + f * nn;
  double* dst = patches + (int64_t(f) * m.n_owned + e) * PATCH_PITCH;

  // ---- copies: 8 loads in flight per lane, coalesced stores
  constexpr int U = 8;
  for (int p0 = 0; p0 < NPATCH; p0 += 32 * U) {
    double v[U];
    int o[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int p = p0 + u * 32 + lane;
      o[u] = p < NPATCH ? soff[p] : -3;
      v[u] = o[u] >= 0 ? __ldg(Ef + o[u]) : 0.0;
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (o[u] >= 0) dst[p0 + u * 32 + lane] = v[u];
  }

  // ---- coarser neighbours: three 1-D sweeps, the thin axis (<= 4 points: the
  // source lies beyond one face of the octant) first, so the scratch is small
  double* es = dyn + warp * WSCR;
  double* t1 = es + NPT + 1;                       // [7][7][n1]
  double* t2 = t1 + T1N;                           // [7][n2][n1]
  const int nc = n_coarse;
  for (int ci = 0; ci < nc; ++ci) {
    const int j = coarse[ci];
    const NbrEntry t = nb[j];
    __syncwarp();                                    // scratch free
    for (int i = lane; i < NPT; i += 32) es[i] = __ldg(Ef + int64_t(t.src) * NPT + i);
    int lo[3], n[3];
#pragma unroll
    for (int k = 0; k < 3; ++k) {
      lo[k] = t.lo[k];
      n[k] = t.hi[k] - t.lo[k] + 1;
    }
    // axis order: a1 = thinnest, then the other two in x, y, z order
    const int a1 = n[0] <= n[1] && n[0] <= n[2] ? 0 : (n[1] <= n[2] ? 1 : 2);
    const int a2 = a1 == 0 ? 1 : 0, a3 = a1 == 2 ? 1 : 2;
    const int n1 = n[a1], n2 = n[a2], n3 = n[a3];
    const int es1 = a1 == 0 ? 1 : (a1 == 1 ? 7 : 49);   // element strides of the axes
    const int es2 = a2 == 0 ? 1 : (a2 == 1 ? 7 : 49);
    const int es3 = a3 == 0 ? 1 : (a3 == 1 ? 7 : 49);
    const int ps1 = a1 == 0 ? 1 : (a1 == 1 ? 13 : 169);  // patch strides
    const int ps2 = a2 == 0 ? 1 : (a2 == 1 ? 13 : 169);
    const int ps3 = a3 == 0 ? 1 : (a3 == 1 ? 13 : 169);
    const int o1 = t.o[a1] + lo[a1], o2 = t.o[a2] + lo[a2], o3 = t.o[a3] + lo[a3];
    const float rn1 = 1.0f / float(n1), rn2 = 1.0f / float(n2);
    __syncwarp();
    // T1[r3][r2][i1] = sum_m W[o1+i1][m] E[m, r2, r3]
    for (int idx = lane; idx < 49 * n1; idx += 32) {
      const int r = fdiv(idx, rn1), i1 = idx - r * n1;       // r = r3 * 7 + r2
      const int r3 = r / 7, r2 = r - r3 * 7;
      const double* row = es + r2 * es2 + r3 * es3;
      const int tt = o1 + i1;
      double v;
      if (tt & 1) {
        const double* w = W + tt * 7;
        v = 0.0;
#pragma unroll
        for (int q = 0; q < 7; ++q) v = fma(w[q], row[q * es1], v);
      } else {
        v = row[(tt >> 1) * es1];
      }
      t1[r * n1 + i1] = v;
    }
    __syncwarp();
    // T2[r3][i2][i1] = sum_m W[o2+i2][m] T1[r3][m][i1]
    for (int idx = lane; idx < 7 * n2 * n1; idx += 32) {
      const int q12 = fdiv(idx, rn1), i1 = idx - q12 * n1;
      const int r3 = fdiv(q12, rn2), i2 = q12 - r3 * n2;
      const int tt = o2 + i2;
      const double* col = t1 + r3 * 7 * n1 + i1;
      double v;
      if (tt & 1) {
        const double* w = W + tt * 7;
        v = 0.0;
#pragma unroll
        for (int q = 0; q < 7; ++q) v = fma(w[q], col[q * n1], v);
      } else {
        v = col[(tt >> 1) * n1];
      }
      t2[(r3 * n2 + i2) * n1 + i1] = v;
    }
    __syncwarp();
    // out[i3][i2][i1] = sum_m W[o3+i3][m] T2[m][i2][i1], for the points j sources
    for (int idx = lane; idx < n3 * n2 * n1; idx += 32) {
      const int q12 = fdiv(idx, rn1), i1 = idx - q12 * n1;
      const int i3 = fdiv(q12, rn2), i2 = q12 - i3 * n2;
      const int p = (lo[a1] + i1) * ps1 + (lo[a2] + i2) * ps2 + (lo[a3] + i3) * ps3;
      if (pm[p] != j) continue;
      const int tt = o3 + i3;
      const double* col = t2 + i2 * n1 + i1;
      double v;
      if (tt & 1) {
        const double* w = W + tt * 7;
        v = 0.0;
#pragma unroll
        for (int q = 0; q < 7; ++q) v = fma(w[q], col[q * n2 * n1], v);
      } else {
        v = col[(tt >> 1) * n2 * n1];
      }
      dst[p] = v;
    }
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

void launch_unzip(const DevMesh& m, const double* E, double* patches, int nf, cudaStream_t s) {
  if (m.n_owned <= 0) return;
  const size_t dyn = size_t(UZ_WARPS) * WSCR * sizeof(double);
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_unzip, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn));
    attr = true;
  }
  k_unzip<<<m.n_owned, UZ_THREADS, dyn, s>>>(m, E, patches, nf);
}

}  // namespace dgr
