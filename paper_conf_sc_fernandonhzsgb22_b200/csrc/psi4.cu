// Gravitational-wave extraction support ("Psi_4 ... expanded
// in spin-weighted spherical harmonics on spherical shells"; readings R33-R36
// of DESIGN.md).  The Weyl scalar itself is the generated
// kernel k_psi4 (gen/psi4.cu); here:
//  * k_octant_xyz: position of every octant node relative to the extraction
//    centre (the tetrad's r^, theta^, phi^ are taken about it);
//  * k_sphere_interp: Psi_4 at extraction-sphere points, each the degree-6
//    tensor Lagrange interpolant of the 343 nodal values of the finest octant
//    containing it (R36), weights l_m(t) = prod_{q != m} (t - q) / (m - q).
#include <cuda_runtime.h>

#include "device.cuh"

namespace dgr {

__global__ void k_octant_xyz(DevMesh m, double cx, double cy, double cz, double* __restrict__ xyz,
                             int64_t ld) {
  const int64_t n = int64_t(m.n_owned) * NPT;
  const double unit = m.width / double(6 * (int64_t(1) << m.D));
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int e = int(i / NPT), p = int(i - int64_t(e) * NPT);
    const int4 o = m.oct[e];
    const int64_t s = int64_t(1) << (m.D - o.w);
    const int64_t X[3] = {6 * int64_t(o.x) + (p % 7) * s, 6 * int64_t(o.y) + ((p / 7) % 7) * s,
                          6 * int64_t(o.z) + (p / 49) * s};
    xyz[i] = m.xmin[0] + double(X[0]) * unit - cx;
    xyz[ld + i] = m.xmin[1] + double(X[1]) * unit - cy;
    xyz[2 * ld + i] = m.xmin[2] + double(X[2]) * unit - cz;
  }
}

void launch_octant_xyz(const DevMesh& m, const double c[3], double* xyz, int64_t ld,
                       cudaStream_t s) {
  if (m.n_owned <= 0) return;
  const int64_t n = int64_t(m.n_owned) * NPT;
  int64_t blocks = (n + 255) / 256;
  if (blocks > int64_t(sm_count()) * 8) blocks = int64_t(sm_count()) * 8;
  k_octant_xyz<<<int(blocks), 256, 0, s>>>(m, c[0], c[1], c[2], xyz, ld);
}

// psi [2][ld] nodal values (column e * 343 + node); point k in octant oct[k]
// at local coordinates t[3][n] (in node units, [0, 6]) -> out [2][n]
__global__ void k_sphere_interp(const double* __restrict__ psi, int64_t ld,
                                const int32_t* __restrict__ oct, const double* __restrict__ t,
                                int64_t n, double* __restrict__ out) {
  for (int64_t k = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; k < n;
       k += int64_t(gridDim.x) * blockDim.x) {
    double w[3][7];
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      const double ta = t[a * n + k];
#pragma unroll
      for (int mm = 0; mm < 7; ++mm) {
        double v = 1.0;
#pragma unroll
        for (int q = 0; q < 7; ++q)
          if (q != mm) v = v * (ta - q) / double(mm - q);
        w[a][mm] = v;
      }
    }
    const double* re = psi + int64_t(oct[k]) * NPT;
    const double* im = re + ld;
    double sr = 0.0, si = 0.0;
    for (int c = 0; c < 7; ++c)
      for (int b = 0; b < 7; ++b) {
        const double wbc = w[2][c] * w[1][b];
#pragma unroll
        for (int a = 0; a < 7; ++a) {
          const int node = a + 7 * b + 49 * c;
          sr = fma(w[0][a] * wbc, re[node], sr);
          si = fma(w[0][a] * wbc, im[node], si);
        }
      }
    out[k] = sr;
    out[n + k] = si;
  }
}

void launch_sphere_interp(const double* psi, int64_t ld, const int32_t* oct, const double* t,
                          int64_t n, double* out, cudaStream_t s) {
  if (n <= 0) return;
  int64_t blocks = (n + 127) / 128;
  if (blocks > int64_t(sm_count()) * 8) blocks = int64_t(sm_count()) * 8;
  k_sphere_interp<<<int(blocks), 128, 0, s>>>(psi, ld, oct, t, n, out);
}

}  // namespace dgr
