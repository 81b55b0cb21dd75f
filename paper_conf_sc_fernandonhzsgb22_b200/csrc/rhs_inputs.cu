// The 234 inputs of the algebraic part A of the BSSN RHS at every interior
// point (§IV-B: 24 values + 72 first + 66 second
// derivatives + 72 Kreiss-Oliger terms), written to HBM — the paper's "easy
// way" (precompute the derivatives in a separate kernel, then combine them in
// A), used to drive the generated A kernels of gen/rhs_alg.cu (the
// Table II study).  Not the default path: k_rhs fuses the
// derivatives with A and never stores them.
//
// One CTA per octant patch of the 13^3 patch buffer, one thread per interior
// point (x fastest); each field patch is staged in shared memory with plain
// coalesced loads and its derivatives evaluated with the stencils of
// readings R8/R10: D1 = (-1,9,-45,0,45,-9,1)/(60h),
// D2 = (2,-27,270,-490,270,-27,2)/(180h^2), mixed = D1 o D1,
// KO_a = sigma/(64h) (1,-6,15,-20,15,-6,1) along a.
// Output layout: in[k][ld], k in codegen/bssn_sym.py's order, column
// e * 343 + p (owned octant e, interior node p).
#include <cuda_runtime.h>

#include "device.cuh"

namespace dgr {

namespace {
constexpr int IT = 352;
__constant__ int c_second_slot[NF] = {0, 1, -1, -1, -1, -1, 2, 3, 4, -1, -1, -1,
                                      5, 6, 7, 8, 9, 10, -1, -1, -1, -1, -1, -1};
}  // namespace

__global__ void __launch_bounds__(IT, 2)
    k_rhs_inputs(DevMesh m, const double* __restrict__ patches, double* __restrict__ in,
                 int64_t ld, double ko_sigma) {
  __shared__ double s[NPATCH];
  const int e = blockIdx.x;
  const int tid = threadIdx.x;
  const int p = tid < NPT ? tid : 0;
  const int c = (p % 7 + 3) + 13 * ((p / 7) % 7 + 3) + 169 * (p / 49 + 3);
  const int4 oi = m.oct[e];
  const double ih = (6.0 * double(int64_t(1) << oi.w)) / m.width;
  const double f1 = ih * (1.0 / 60.0), f2 = ih * ih * (1.0 / 180.0), fm = ih * ih * (1.0 / 3600.0);
  const double kos = ko_sigma * ih * (1.0 / 64.0);
  const int64_t col = int64_t(e) * NPT + p;
  const int64_t fstride = int64_t(m.n_owned) * PATCH_PITCH;
  for (int f = 0; f < NF; ++f) {
    const double* src = patches + f * fstride + int64_t(e) * PATCH_PITCH;
    __syncthreads();
    for (int k = tid; k < NPATCH; k += IT) s[k] = src[k];
    __syncthreads();
    if (tid >= NPT) continue;
    in[f * ld + col] = s[c];
    const int st[3] = {1, 13, 169};
    double d2[3];
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      const int q = st[a];
      const double u0 = s[c], a1 = s[c + q], b1 = s[c - q], a2 = s[c + 2 * q], b2 = s[c - 2 * q],
                   a3 = s[c + 3 * q], b3 = s[c - 3 * q];
      in[(24 + 3 * f + a) * ld + col] = ((a1 - b1) * 45.0 - (a2 - b2) * 9.0 + (a3 - b3)) * f1;
      const double s1 = a1 + b1, s2 = a2 + b2, s3 = a3 + b3;
      d2[a] = (2.0 * s3 - 27.0 * s2 + 270.0 * s1 - 490.0 * u0) * f2;
      in[(162 + 3 * f + a) * ld + col] = (s3 - 6.0 * s2 + 15.0 * s1 - 20.0 * u0) * kos;
    }
    const int ss = c_second_slot[f];
    if (ss >= 0) {
      auto mixed = [&](int sa, int sb) {
        double r[7];
#pragma unroll
        for (int b = -3; b <= 3; ++b) {
          const int cb = c + b * sb;
          r[b + 3] = (s[cb + sa] - s[cb - sa]) * 45.0 - (s[cb + 2 * sa] - s[cb - 2 * sa]) * 9.0 +
                     (s[cb + 3 * sa] - s[cb - 3 * sa]);
        }
        return ((r[4] - r[2]) * 45.0 - (r[5] - r[1]) * 9.0 + (r[6] - r[0])) * fm;
      };
      double* o = in + (96 + 6 * ss) * ld + col;
      o[0 * ld] = d2[0];
      o[1 * ld] = mixed(1, 13);
      o[2 * ld] = mixed(1, 169);
      o[3 * ld] = d2[1];
      o[4 * ld] = mixed(13, 169);
      o[5 * ld] = d2[2];
    }
  }
}

void launch_rhs_inputs(const DevMesh& m, const double* patches, double* in, int64_t ld,
                       double ko_sigma, cudaStream_t s) {
  if (m.n_owned <= 0) return;
  k_rhs_inputs<<<m.n_owned, IT, 0, s>>>(m, patches, in, ld, ko_sigma);
}

}  // namespace dgr
