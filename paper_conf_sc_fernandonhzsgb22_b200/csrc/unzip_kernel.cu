// Octant-to-patch ("unzip"), Alg. 2 (L249-283) / §IV-A (L235-306).
//
// Gather formulation: one CTA per (patch, chunk of 4 fields).
// At CTA start the per-point source offsets are resolved once into shared
// memory (copy from self / same-level / finer neighbours = one load of a
// reconstructed nodal value, their half-grid coordinates being even).  Per
// field: all copy loads and the 7^3 nodal values of the coarser neighbours are
// issued together, then each coarser neighbour's points are produced by three
// 1-D degree-6 Lagrange sweeps (x -> y -> z) restricted to the bounding box of
// the points it sources (tensor-product interpolation), then the
// outer-boundary extrapolation (reading R12), then the 13^3 patch leaves with
// streaming 16-B stores (st.global.cs keeps the element buffer in L2).
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
constexpr int UZ_THREADS = 256;
constexpr int UZ_FCHUNK = 4;                                  // fields per CTA
constexpr int PER = (NPATCH + UZ_THREADS - 1) / UZ_THREADS;   // 9 points per thread
constexpr int UZ_MAXC = 3;                                    // coarse sources staged at once
constexpr int EPER = (UZ_MAXC * NPT + UZ_THREADS - 1) / UZ_THREADS;
constexpr int BOXMAX = 10;                                    // coarse-source box edge <= 10

// q = floor(i / n) for 0 <= i < 2^16, 1 <= n <= 13 (float reciprocal, exact here)
__device__ __forceinline__ int fdiv(int i, float rn) { return int((float(i) + 0.5f) * rn); }
}  // namespace

__global__ void __launch_bounds__(UZ_THREADS) k_unzip(DevMesh m, const double* __restrict__ E,
                                                      double* __restrict__ patches, int nf) {
  __shared__ __align__(16) double P[NPATCH + 3];
  __shared__ __align__(16) uint8_t pm[PMAP_PITCH];
  __shared__ int32_t soff[NPATCH];
  __shared__ double Es[UZ_MAXC][NPT + 1];
  __shared__ double T1[49 * BOXMAX];
  __shared__ double T2[7 * BOXMAX * BOXMAX];
  __shared__ NbrEntry nb[NBR_MAX];
  __shared__ double W[91];
  __shared__ double WX[21];
  __shared__ int coarse[8];
  __shared__ int n_coarse;
  const int e = blockIdx.x;
  const int tid = threadIdx.x;
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
  // resolve every point's source once (element-buffer offset, -1: computed later)
  for (int p = tid; p < NPATCH; p += UZ_THREADS) {
    const int j = pm[p];
    const int ix = p % 13, iy = (p / 13) % 13, iz = p / 169;
    int off = -1;
    if (j == PM_SELF) {
      off = e * NPT + (ix - 3) + 7 * (iy - 3) + 49 * (iz - 3);
    } else if (j != PM_EXTRAP && nb[j].r != 1) {
      const NbrEntry& t = nb[j];
      const int tx = (t.o[0] + t.r * ix) >> 1, ty = (t.o[1] + t.r * iy) >> 1,
                tz = (t.o[2] + t.r * iz) >> 1;
      off = t.src * NPT + tx + 7 * ty + 49 * tz;
    }
    soff[p] = off;
  }
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
  const int nc0 = nc < UZ_MAXC ? nc : UZ_MAXC;
  const int64_t nn = int64_t(m.n_local) * NPT;
  const int f0 = blockIdx.y * UZ_FCHUNK, f1 = min(nf, f0 + UZ_FCHUNK);
  for (int f = f0; f < f1; ++f) {
    const double* Ef = E + f * nn;
    // ---- copies + coarse nodal values: every load in flight together
    {
      double v[PER], ev[EPER];
      int off[PER];
#pragma unroll
      for (int q = 0; q < PER; ++q) {
        const int p = tid + q * UZ_THREADS;
        off[q] = p < NPATCH ? soff[p] : -1;
      }
#pragma unroll
      for (int q = 0; q < PER; ++q) v[q] = off[q] >= 0 ? __ldg(Ef + off[q]) : 0.0;
#pragma unroll
      for (int q = 0; q < EPER; ++q) {
        const int i = tid + q * UZ_THREADS;
        ev[q] = 0.0;
        if (i < nc0 * NPT) {
          const int c = i / NPT;
          ev[q] = __ldg(Ef + int64_t(nb[coarse[c]].src) * NPT + (i - c * NPT));
        }
      }
#pragma unroll
      for (int q = 0; q < PER; ++q)
        if (off[q] >= 0) P[tid + q * UZ_THREADS] = v[q];
#pragma unroll
      for (int q = 0; q < EPER; ++q) {
        const int i = tid + q * UZ_THREADS;
        if (i < nc0 * NPT) {
          const int c = i / NPT;
          Es[c][i - c * NPT] = ev[q];
        }
      }
    }
    // ---- coarser neighbours: separable sweeps x -> y -> z
    for (int ci = 0; ci < nc; ++ci) {
      const int j = coarse[ci];
      const NbrEntry t = nb[j];
      const int slot = ci % UZ_MAXC;
      if (ci >= UZ_MAXC) {  // rare: more than UZ_MAXC coarser neighbours
        __syncthreads();
        for (int i = tid; i < NPT; i += UZ_THREADS)
          Es[slot][i] = __ldg(Ef + int64_t(t.src) * NPT + i);
      }
      __syncthreads();
      const int lx = t.lo[0], ly = t.lo[1], lz = t.lo[2];
      const int nx = t.hi[0] - lx + 1, ny = t.hi[1] - ly + 1, nz = t.hi[2] - lz + 1;
      const float rnx = 1.0f / float(nx), rny = 1.0f / float(ny);
      const double* es = Es[slot];
      for (int idx = tid; idx < 49 * nx; idx += UZ_THREADS) {
        const int cyz = fdiv(idx, rnx), ix = idx - cyz * nx;     // cyz = cz * 7 + cy
        const int tx = t.o[0] + lx + ix;
        const double* row = es + cyz * 7;
        double v;
        if (tx & 1) {
          const double* w = W + tx * 7;
          v = 0.0;
#pragma unroll
          for (int a = 0; a < 7; ++a) v = fma(w[a], row[a], v);
        } else {
          v = row[tx >> 1];
        }
        T1[cyz * BOXMAX + ix] = v;
      }
      __syncthreads();
      for (int idx = tid; idx < 7 * ny * nx; idx += UZ_THREADS) {
        const int q1 = fdiv(idx, rnx), ix = idx - q1 * nx;
        const int cz = fdiv(q1, rny), iy = q1 - cz * ny;
        const int ty = t.o[1] + ly + iy;
        double v;
        if (ty & 1) {
          const double* w = W + ty * 7;
          v = 0.0;
#pragma unroll
          for (int b = 0; b < 7; ++b) v = fma(w[b], T1[(cz * 7 + b) * BOXMAX + ix], v);
        } else {
          v = T1[(cz * 7 + (ty >> 1)) * BOXMAX + ix];
        }
        T2[(cz * BOXMAX + iy) * BOXMAX + ix] = v;
      }
      __syncthreads();
      for (int idx = tid; idx < nz * ny * nx; idx += UZ_THREADS) {
        const int q1 = fdiv(idx, rnx), ix = idx - q1 * nx;
        const int iz = fdiv(q1, rny), iy = q1 - iz * ny;
        const int p = (lx + ix) + 13 * (ly + iy) + 169 * (lz + iz);
        if (pm[p] != j) continue;
        const int tz = t.o[2] + lz + iz;
        double v;
        if (tz & 1) {
          const double* w = W + tz * 7;
          v = 0.0;
#pragma unroll
          for (int c = 0; c < 7; ++c) v = fma(w[c], T2[(c * BOXMAX + iy) * BOXMAX + ix], v);
        } else {
          v = T2[((tz >> 1) * BOXMAX + iy) * BOXMAX + ix];
        }
        P[p] = v;
      }
    }
    // ---- phase B: extrapolation along x, then y, then z (reading R12), slabs only
    if (any_out) {
      for (int a = 0; a < 3; ++a) {
        __syncthreads();
        const int sa = a == 0 ? 1 : (a == 1 ? 13 : 169);
        const int sb = a == 0 ? 13 : 1, sc = a == 2 ? 13 : 169;   // the two other axes
        const int b_ax = a == 0 ? 1 : 0, c_ax = a == 2 ? 1 : 2;
        for (int side = 0; side < 2; ++side) {
          if (!(side == 0 ? out_lo[a] : out_hi[a])) continue;
          for (int idx = tid; idx < 3 * 169; idx += UZ_THREADS) {
            const int k3 = idx % 3, uv = idx / 3;
            const int cb = uv % 13, cc = uv / 13;   // indices along axes b_ax, c_ax
            // only points inside along every later axis
            bool later_in = true;
            if (b_ax > a && ((cb < 3 && out_lo[b_ax]) || (cb > 9 && out_hi[b_ax]))) later_in = false;
            if (c_ax > a && ((cc < 3 && out_lo[c_ax]) || (cc > 9 && out_hi[c_ax]))) later_in = false;
            if (!later_in) continue;
            const int ia = side == 0 ? k3 : 10 + k3;
            const int base = cb * sb + cc * sc;
            const int p = base + ia * sa;
            double acc = 0.0;
            if (side == 0) {
              const double* w = WX + (2 - ia) * 7;       // t = -(3 - ia)
#pragma unroll
              for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], P[base + (3 + mm) * sa], acc);
            } else {
              const double* w = WX + (ia - 10) * 7;      // mirrored
#pragma unroll
              for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], P[base + (9 - mm) * sa], acc);
            }
            P[p] = acc;
          }
        }
      }
    }
    __syncthreads();
    double* dst = patches + (int64_t(f) * m.n_owned + e) * PATCH_PITCH;
    const double2* P2 = reinterpret_cast<const double2*>(P);
    double2* d2 = reinterpret_cast<double2*>(dst);
    for (int i = tid; i < NPATCH / 2; i += UZ_THREADS) __stcs(d2 + i, P2[i]);
    if (tid == 0) __stcs(dst + NPATCH - 1, P[NPATCH - 1]);
    __syncthreads();
  }
}

void launch_unzip(const DevMesh& m, const double* E, double* patches, int nf, cudaStream_t s) {
  if (m.n_owned <= 0) return;
  k_unzip<<<dim3(m.n_owned, (nf + UZ_FCHUNK - 1) / UZ_FCHUNK), UZ_THREADS, 0, s>>>(m, E, patches,
                                                                                  nf);
}

}  // namespace dgr
