// Regrid kernels (Alg. 1 line 3 construct_grid,
// P:L198-215, refinement tolerance P:L465; readings R30-R32 of DESIGN.md):
//  * k_wavelet: per owned octant, the wavelet refinement indicator — the
//    largest |P - prediction| over the interior points of its 13^3 patches of
//    the selected fields, the prediction being the tensor degree-6 Lagrange
//    interpolant from the all-even patch points (spacing 2h; R30);
//  * k_transfer: every DOF of the new mesh takes the old mesh's piecewise
//    interpolant at its position — the tensor Lagrange interpolant of the
//    finest old element containing it, at half-grid coordinates t2 (R32).
#include <cuda_runtime.h>

#include "device.cuh"

namespace dgr {

namespace {
constexpr int WT = 352;
__constant__ double c_gW13[13 * 7];   // l_m(t2 / 2), rows t2 = 0..12 (host-computed, exact)
}  // namespace

void upload_regrid_tables(const double* w13) {
  cudaMemcpyToSymbol(c_gW13, w13, sizeof(double) * 91);
}

// one CTA per owned octant; thread p < 343 owns interior point p
__global__ void __launch_bounds__(WT)
    k_wavelet(DevMesh m, const double* __restrict__ patches, uint32_t mask, double* __restrict__ w) {
  __shared__ double s[NPATCH];
  __shared__ double red[WT / 32];
  const int e = blockIdx.x, tid = threadIdx.x;
  const int p = tid < NPT ? tid : 0;
  const int ix = p % 7 + 3, iy = (p / 7) % 7 + 3, iz = p / 49 + 3;   // patch indices 3..9
  const int64_t fstride = int64_t(m.n_owned) * PATCH_PITCH;
  double wmax = 0.0;
  for (int f = 0; f < NF; ++f) {
    if (!((mask >> f) & 1u)) continue;
    const double* src = patches + f * fstride + int64_t(e) * PATCH_PITCH;
    __syncthreads();
    for (int k = tid; k < NPATCH; k += WT) s[k] = src[k];
    __syncthreads();
    if (tid >= NPT) continue;
    // rows over the even points m (patch index 2m) for each axis: a single
    // unit term at an even index, the 7 weights l_m(i/2) at an odd one
    const int na = (ix & 1) ? 7 : 1, nb = (iy & 1) ? 7 : 1, nc = (iz & 1) ? 7 : 1;
    const int a0 = (ix & 1) ? 0 : ix / 2, b0 = (iy & 1) ? 0 : iy / 2, c0 = (iz & 1) ? 0 : iz / 2;
    double pred = 0.0;
    for (int c = 0; c < nc; ++c) {
      const double wc = (iz & 1) ? c_gW13[iz * 7 + c] : 1.0;
      double sy = 0.0;
      for (int b = 0; b < nb; ++b) {
        const double wb = (iy & 1) ? c_gW13[iy * 7 + b] : 1.0;
        double sx = 0.0;
        for (int a = 0; a < na; ++a) {
          const double wa = (ix & 1) ? c_gW13[ix * 7 + a] : 1.0;
          sx = fma(wa, s[2 * (a0 + a) + 13 * 2 * (b0 + b) + 169 * 2 * (c0 + c)], sx);
        }
        sy = fma(wb, sx, sy);
      }
      pred = fma(wc, sy, pred);
    }
    wmax = fmax(wmax, fabs(s[ix + 13 * iy + 169 * iz] - pred));
  }
  if (tid >= NPT) wmax = 0.0;
  for (int o = 16; o > 0; o >>= 1) wmax = fmax(wmax, __shfl_xor_sync(0xffffffffu, wmax, o));
  if ((tid & 31) == 0) red[tid >> 5] = wmax;
  __syncthreads();
  if (tid == 0) {
    double r = 0.0;
    for (int k = 0; k < WT / 32; ++k) r = fmax(r, red[k]);
    w[e] = r;
  }
}

void launch_wavelet(const DevMesh& m, const double* patches, uint32_t mask, double* w,
                    cudaStream_t s) {
  if (m.n_owned <= 0) return;
  k_wavelet<<<m.n_owned, WT, 0, s>>>(m, patches, mask, w);
}

// map[i] = {old local element, t2x | t2y << 8 | t2z << 16, -, -} for new DOF i
__global__ void k_transfer(DevMesh old, const double* __restrict__ u_old, const int4* __restrict__ map,
                           int64_t n, double* __restrict__ u_new, int64_t new_stride) {
  const int64_t ds = old.dof_stride;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int4 q = map[i];
    const int t2[3] = {q.y & 255, (q.y >> 8) & 255, (q.y >> 16) & 255};
    const int na = (t2[0] & 1) ? 7 : 1, nb = (t2[1] & 1) ? 7 : 1, nc = (t2[2] & 1) ? 7 : 1;
    const int a0 = (t2[0] & 1) ? 0 : t2[0] / 2, b0 = (t2[1] & 1) ? 0 : t2[1] / 2,
              c0 = (t2[2] & 1) ? 0 : t2[2] / 2;
    const int32_t* o2s = old.o2s + int64_t(q.x) * NPT;
    for (int f = 0; f < NF; ++f) {
      const double* uf = u_old + f * ds;
      const double* af = old.aux + f * old.aux_stride - ds;
      double v = 0.0;
      for (int c = 0; c < nc; ++c) {
        const double wc = (t2[2] & 1) ? c_gW13[t2[2] * 7 + c] : 1.0;
        double sy = 0.0;
        for (int b = 0; b < nb; ++b) {
          const double wb = (t2[1] & 1) ? c_gW13[t2[1] * 7 + b] : 1.0;
          double sx = 0.0;
          for (int a = 0; a < na; ++a) {
            const double wa = (t2[0] & 1) ? c_gW13[t2[0] * 7 + a] : 1.0;
            const int32_t x = __ldg(o2s + (a0 + a) + 7 * (b0 + b) + 49 * (c0 + c));
            sx = fma(wa, x < ds ? __ldg(uf + x) : af[x], sx);
          }
          sy = fma(wb, sx, sy);
        }
        v = fma(wc, sy, v);
      }
      u_new[f * new_stride + i] = v;
    }
  }
}

void launch_transfer(const DevMesh& old, const double* u_old, const int4* map, int64_t n,
                     double* u_new, int64_t new_stride, cudaStream_t s) {
  if (n <= 0) return;
  int64_t blocks = (n + 127) / 128;
  const int64_t cap = int64_t(sm_count()) * 16;
  if (blocks > cap) blocks = cap;
  k_transfer<<<int(blocks), 128, 0, s>>>(old, u_old, map, n, u_new, new_stride);
}

}  // namespace dgr
