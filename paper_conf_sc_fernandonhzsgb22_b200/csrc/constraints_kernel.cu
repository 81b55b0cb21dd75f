// Constraint diagnostics (not in the paper; BASELINE.json north_star asks for
// dgr_constraints): H, M^i, G^i at the interior points of every patch,
//   H   = chi gt^ij R_ij + 2/3 K^2 - At_ij At^ij
//   M^i = d_j At^ij + Gt^i_jk At^jk - 2/3 gt^ij d_j K - 3/(2 chi) At^ij d_j chi
//   G^i = Gt^i - gt^jk Gt^i_jk
// Same staging scheme as the RHS kernel (one CTA per patch, fields streamed
// through shared memory by TMA bulk copies, per-point state in smem slots).
// Exact simplifications: gt^ij of the d Gt part of Rt_ij is d_k Gt^k, and
// gt^ij gt_ij = 3 in the trace of R^chi.
#include <cuda_runtime.h>

#include "device.cuh"

namespace dgr {

namespace {

constexpr int CT = 352;
constexpr int NPP = 344;
constexpr int V_GT = 0, V_GAM = 3, V_AT = 9;  // values (15)
constexpr int G_INV = 15;                     // 6
constexpr int S0 = 21;                        // 24 scratch
constexpr int ACC = 45;                       // H, M0..2  (4)
constexpr int NSLOT = 49;
constexpr int NFC = 17;
constexpr size_t SMEM_BYTES = size_t(NSLOT) * NPP * 8 + size_t(2) * STAGE_DBL * 8 + 16;

// gt_ij (6) -> [Christoffel block] -> chi -> K -> At_ij (6) -> Gt^i (3)
__constant__ int c_corder[NFC] = {12, 13, 14, 15, 16, 17, 1, 2, 18, 19, 20, 21, 22, 23, 3, 4, 5};

__device__ __forceinline__ int sidx(int i, int j) {
  return i <= j ? (i == 0 ? j : (i == 1 ? 2 + j : 5)) : (j == 0 ? i : (j == 1 ? 2 + i : 5));
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void bulk_load(double* dst, const double* src, uint32_t bytes,
                                          uint64_t* bar) {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
        " selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}
__device__ __forceinline__ double d1_at(const double* s, int c, int st) {
  return (s[c + st] - s[c - st]) * 45.0 - (s[c + 2 * st] - s[c - 2 * st]) * 9.0 +
         (s[c + 3 * st] - s[c - 3 * st]);
}
__device__ __forceinline__ double d2_at(const double* s, int c, int st) {
  return 2.0 * (s[c + 3 * st] + s[c - 3 * st]) - 27.0 * (s[c + 2 * st] + s[c - 2 * st]) +
         270.0 * (s[c + st] + s[c - st]) - 490.0 * s[c];
}
__device__ __forceinline__ double mixed(const double* s, int c, int sa, int sb) {
  double r[7];
#pragma unroll
  for (int b = -3; b <= 3; ++b) {
    if (b == 0) continue;
    r[b + 3] = d1_at(s, c + b * sb, sa);
  }
  return (r[4] - r[2]) * 45.0 - (r[5] - r[1]) * 9.0 + (r[6] - r[0]);
}
__device__ __forceinline__ double trace6(const double* gi, const double* X) {
  return gi[0] * X[0] + gi[3] * X[3] + gi[5] * X[5] +
         2.0 * (gi[1] * X[1] + gi[2] * X[2] + gi[4] * X[4]);
}

}  // namespace

// (__maxnreg__(184) removes half the spills but the launch then fails with
// "too many resources requested": kept at __launch_bounds__(352, 1))
__global__ void __launch_bounds__(CT, 1)
    k_constraints(DevMesh m, const double* __restrict__ patches, double* __restrict__ c_oct,
                  RhsParams prm) {
  extern __shared__ __align__(128) double smem[];
  double* slots = smem;
  double* stage = smem + NSLOT * NPP;
  uint64_t* bars = reinterpret_cast<uint64_t*>(stage + 2 * STAGE_DBL);
  const int e = blockIdx.x;
  const int tid = threadIdx.x;
  const bool active = tid < NPT;
  const int p = active ? tid : 0;
  const int c0 = (p % 7 + 3) + 13 * ((p / 7) % 7 + 3) + 169 * (p / 49 + 3);
  const int64_t no = m.n_owned;
  const double* pbase = patches + int64_t(e) * PATCH_PITCH;
  const int64_t fstride = no * PATCH_PITCH;
#define SL(slot) slots[(slot) * NPP + p]
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[0])));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[1])));
  }
  __syncthreads();
  if (tid == 0) {
    bulk_load(stage, pbase + c_corder[0] * fstride, STAGE_DBL * 8, &bars[0]);
    bulk_load(stage + STAGE_DBL, pbase + c_corder[1] * fstride, STAGE_DBL * 8, &bars[1]);
  }
  const int4 oi = m.oct[e];
  const double ih = (6.0 * double(int64_t(1) << oi.w)) / m.width;
  const double f1 = ih * (1.0 / 60.0), f2 = ih * ih * (1.0 / 180.0), fm = ih * ih * (1.0 / 3600.0);
  double chi = 0, Kv = 0;
  if (active) {
    chi = __ldg(pbase + 1 * fstride + c0);
    Kv = __ldg(pbase + 2 * fstride + c0);
    for (int i = 0; i < 3; ++i) SL(V_GT + i) = __ldg(pbase + (3 + i) * fstride + c0);
    double g[6];
    for (int q = 0; q < 6; ++q) {
      g[q] = __ldg(pbase + (12 + q) * fstride + c0);
      SL(V_GAM + q) = g[q];
      SL(V_AT + q) = __ldg(pbase + (18 + q) * fstride + c0);
    }
    const double a00 = g[3] * g[5] - g[4] * g[4];
    const double a01 = g[2] * g[4] - g[1] * g[5];
    const double a02 = g[1] * g[4] - g[2] * g[3];
    const double idet = 1.0 / (g[0] * a00 + g[1] * a01 + g[2] * a02);
    SL(G_INV + 0) = a00 * idet;
    SL(G_INV + 1) = a01 * idet;
    SL(G_INV + 2) = a02 * idet;
    SL(G_INV + 3) = (g[0] * g[5] - g[2] * g[2]) * idet;
    SL(G_INV + 4) = (g[1] * g[2] - g[0] * g[4]) * idet;
    SL(G_INV + 5) = (g[0] * g[3] - g[1] * g[1]) * idet;
    for (int q = 0; q < 4; ++q) SL(ACC + q) = 0.0;
  }
  const double ichi = 1.0 / fmax(chi, prm.chi_floor);
  double Au[6] = {0, 0, 0, 0, 0, 0};
  for (int st = 0; st < NFC; ++st) {
    const int buf = st & 1;
    mbar_wait(&bars[buf], (st >> 1) & 1);
    const double* s = stage + buf * STAGE_DBL;
    const int f = c_corder[st];
    if (active) {
      double gi[6];
#pragma unroll
      for (int r = 0; r < 6; ++r) gi[r] = SL(G_INV + r);
      const double d1[3] = {d1_at(s, c0, 1) * f1, d1_at(s, c0, 13) * f1, d1_at(s, c0, 169) * f1};
      if (f >= 12 && f <= 17) {
        const int q = f - 12;
        double dd[6];
        dd[0] = d2_at(s, c0, 1) * f2;
        dd[3] = d2_at(s, c0, 13) * f2;
        dd[5] = d2_at(s, c0, 169) * f2;
        dd[1] = mixed(s, c0, 1, 13) * fm;
        dd[2] = mixed(s, c0, 1, 169) * fm;
        dd[4] = mixed(s, c0, 13, 169) * fm;
        for (int k = 0; k < 3; ++k) SL(S0 + k * 6 + q) = d1[k];
        SL(S0 + 18 + q) = trace6(gi, dd);
        if (q == 5) {
          double At[6];
          for (int r = 0; r < 6; ++r) At[r] = SL(V_AT + r);
          double C[3][6], Gam[3][6], cal[3];
#pragma unroll
          for (int k = 0; k < 3; ++k)
#pragma unroll
            for (int i = 0; i < 3; ++i)
#pragma unroll
              for (int j = i; j < 3; ++j)
                C[k][sidx(i, j)] = 0.5 * (SL(S0 + i * 6 + sidx(k, j)) +
                                          SL(S0 + j * 6 + sidx(k, i)) - SL(S0 + k * 6 + sidx(i, j)));
#pragma unroll
          for (int k = 0; k < 3; ++k)
#pragma unroll
            for (int q2 = 0; q2 < 6; ++q2)
              Gam[k][q2] = gi[sidx(k, 0)] * C[0][q2] + gi[sidx(k, 1)] * C[1][q2] +
                           gi[sidx(k, 2)] * C[2][q2];
#pragma unroll
          for (int k = 0; k < 3; ++k) cal[k] = trace6(gi, Gam[k]);
          // trace of Rt without the d Gt term
          double trR = 0.0;
#pragma unroll
          for (int i = 0; i < 3; ++i)
#pragma unroll
            for (int j = 0; j < 3; ++j) {
              double r = -0.5 * SL(S0 + 18 + sidx(i, j));
              double c2 = 0.0;
              for (int k = 0; k < 3; ++k) c2 += cal[k] * (C[i][sidx(j, k)] + C[j][sidx(i, k)]);
              r += 0.5 * c2;
              double qs = 0.0;
#pragma unroll
              for (int l = 0; l < 3; ++l)
#pragma unroll
                for (int mm = 0; mm < 3; ++mm) {
                  double t = 0.0;
#pragma unroll
                  for (int k = 0; k < 3; ++k)
                    t += Gam[k][sidx(l, i)] * C[j][sidx(k, mm)] +
                         Gam[k][sidx(l, j)] * C[i][sidx(k, mm)] +
                         Gam[k][sidx(i, mm)] * C[k][sidx(l, j)];
                  qs += gi[sidx(l, mm)] * t;
                }
              trR += gi[sidx(i, j)] * (r + qs);
            }
          SL(ACC + 0) += chi * trR;
          // At^ij
#pragma unroll
          for (int i = 0; i < 3; ++i)
#pragma unroll
            for (int j = i; j < 3; ++j) {
              double a = 0.0;
              for (int k = 0; k < 3; ++k)
                for (int l = 0; l < 3; ++l) a += gi[sidx(i, k)] * gi[sidx(j, l)] * At[sidx(k, l)];
              Au[sidx(i, j)] = a;
            }
          // M^i: Gt^i_jk At^jk + chain-rule part of d_j At^ij
          //   d_j gt^ik = -(Gt^i_jm gt^mk + Gt^k_jm gt^mi)
          for (int i = 0; i < 3; ++i) {
            double v = trace6(Au, Gam[i]);
            for (int j = 0; j < 3; ++j)
              for (int k = 0; k < 3; ++k) {
                double dgik = 0.0, dgjk = 0.0;
                for (int mm = 0; mm < 3; ++mm) {
                  dgik -= Gam[i][sidx(j, mm)] * gi[sidx(mm, k)] + Gam[k][sidx(j, mm)] * gi[sidx(mm, i)];
                  dgjk -= Gam[j][sidx(j, mm)] * gi[sidx(mm, k)] + Gam[k][sidx(j, mm)] * gi[sidx(mm, j)];
                }
                // (d_j gt^ik) gt^jl At_kl + gt^ik (d_j gt^jl) At_kl  (here k plays l in the 2nd)
                double Ajk = 0.0, Aik = 0.0;
                for (int l = 0; l < 3; ++l) {
                  Ajk += gi[sidx(j, l)] * At[sidx(k, l)];
                  Aik += gi[sidx(i, l)] * At[sidx(l, k)];
                }
                v += dgik * Ajk + dgjk * Aik;
              }
            SL(ACC + 1 + i) += v;
          }
          // G^i = Gt^i - CalGt^i ; keep Gt^k_ij and CalGt^k
          for (int k = 0; k < 3; ++k)
            for (int q2 = 0; q2 < 6; ++q2) SL(S0 + k * 6 + q2) = Gam[k][q2];
          for (int k = 0; k < 3; ++k) SL(S0 + 18 + k) = cal[k];
        }
      } else if (f == 1) {
        double dd[6];
        dd[0] = d2_at(s, c0, 1) * f2;
        dd[3] = d2_at(s, c0, 13) * f2;
        dd[5] = d2_at(s, c0, 169) * f2;
        dd[1] = mixed(s, c0, 1, 13) * fm;
        dd[2] = mixed(s, c0, 1, 169) * fm;
        dd[4] = mixed(s, c0, 13, 169) * fm;
        // trace of R^chi (eqs 18-19): gt^ij[(d_ij chi - Gt^k_ij d_k chi)/(2chi) - d_i chi d_j chi/(4chi^2)]
        //   + 3/(2chi)[gt^kl(d_kl chi - 3/(2chi) d_k chi d_l chi) - CalGt^m d_m chi]
        double Rc[6];
        for (int i = 0; i < 3; ++i)
          for (int j = i; j < 3; ++j) {
            const int q = sidx(i, j);
            const double gd = SL(S0 + q) * d1[0] + SL(S0 + 6 + q) * d1[1] + SL(S0 + 12 + q) * d1[2];
            Rc[q] = (dd[q] - gd) * (0.5 * ichi) - d1[i] * d1[j] * (0.25 * ichi * ichi);
          }
        double dchi2[6];
        for (int i = 0; i < 3; ++i)
          for (int j = i; j < 3; ++j) dchi2[sidx(i, j)] = d1[i] * d1[j];
        const double calc = SL(S0 + 18) * d1[0] + SL(S0 + 19) * d1[1] + SL(S0 + 20) * d1[2];
        const double trRc = trace6(gi, Rc) +
                            1.5 * ichi * (trace6(gi, dd) - 1.5 * ichi * trace6(gi, dchi2) - calc);
        SL(ACC + 0) += chi * trRc;
        for (int i = 0; i < 3; ++i)
          SL(ACC + 1 + i) -= 1.5 * ichi *
                             (Au[sidx(i, 0)] * d1[0] + Au[sidx(i, 1)] * d1[1] + Au[sidx(i, 2)] * d1[2]);
      } else if (f == 2) {
        for (int i = 0; i < 3; ++i)
          SL(ACC + 1 + i) -= (2.0 / 3.0) * (gi[sidx(i, 0)] * d1[0] + gi[sidx(i, 1)] * d1[1] +
                                            gi[sidx(i, 2)] * d1[2]);
      } else if (f >= 18) {
        // gt^ik gt^jl d_j At_kl for the (k,l) = q component (both orders if k != l)
        const int q = f - 18;
        const int kq = q < 3 ? 0 : (q < 5 ? 1 : 2);
        const int lq = q < 3 ? q : (q < 5 ? q - 2 : 2);
        for (int i = 0; i < 3; ++i) {
          double v = 0.0;
          for (int j = 0; j < 3; ++j) {
            double w = gi[sidx(i, kq)] * gi[sidx(j, lq)];
            if (kq != lq) w += gi[sidx(i, lq)] * gi[sidx(j, kq)];
            v += w * d1[j];
          }
          SL(ACC + 1 + i) += v;
        }
      } else if (f >= 3 && f <= 5) {
        // chi gt^ij (d Gt part of Rt) = chi d_k Gt^k
        SL(ACC + 0) += chi * d1[f - 3];
      }
    }
    __syncthreads();
    if (tid == 0 && st + 2 < NFC)
      bulk_load(stage + buf * STAGE_DBL, pbase + c_corder[st + 2] * fstride, STAGE_DBL * 8,
                &bars[buf]);
  }
  if (active) {
    double At[6];
    for (int r = 0; r < 6; ++r) At[r] = SL(V_AT + r);
    const double AA = At[0] * Au[0] + At[3] * Au[3] + At[5] * Au[5] +
                      2.0 * (At[1] * Au[1] + At[2] * Au[2] + At[4] * Au[4]);
    double* out = c_oct + int64_t(e) * NPT + p;
    const int64_t ostr = no * NPT;
    out[0] = SL(ACC + 0) + (2.0 / 3.0) * Kv * Kv - AA;
    for (int i = 0; i < 3; ++i) out[(1 + i) * ostr] = SL(ACC + 1 + i);
    for (int i = 0; i < 3; ++i) out[(4 + i) * ostr] = SL(V_GT + i) - SL(S0 + 18 + i);
  }
#undef SL
}

void launch_constraints(const DevMesh& m, const double* patches, double* c_oct,
                        const RhsParams& p, cudaStream_t s) {
  if (m.n_owned <= 0) return;
  static std::atomic<bool> done[MAX_DEVICES];
  if (first_on_device(done))
    cudaFuncSetAttribute(k_constraints, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(SMEM_BYTES));
  k_constraints<<<m.n_owned, CT, SMEM_BYTES, s>>>(m, patches, c_oct, p);
}

}  // namespace dgr
