// Shared pieces of the RHS kernels (rhs_kernel.cu, rhs_kernel_fi.cu): constants,
// device tables, stencil / tensor helpers, tensor-memory helpers.  Included by
// both translation units; everything is in an anonymous namespace, so each
// has its own copy of the device tables (each uploads them: upload_tables_here).
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <vector>

#include "device.cuh"

namespace dgr {

namespace {

constexpr int RT = 352;   // threads (11 warps); 343 interior points
constexpr int NPP = RT;   // slot stride in doubles: slots are indexed by thread

// shared-memory slot map ([slot][NPP] doubles, indexed by thread).  Slot
// reuse: during the gt stages the A_AT slots hold gt^lm d_lm gt_ij (A_AT is
// first written by the Christoffel block) and from the Christoffel block to the
// beta stages the A_B slots hold CalGt^k (A_B is first written by the B stage).
constexpr int A_GT = 0, A_BETA = 3, A_B = 6, A_GAM = 9, A_AT = 15;             // accumulators (21)
constexpr int S0 = 21;                                                         // scratch (18)
constexpr int NSLOT = 39;
// The point's read-only values live in tensor memory (tm_* below; DESIGN.md
// §7: a thread's TMEM lane is a private store outside the shared-memory data
// pipe), 6 doubles per block: TV_GT gt_ij, TV_AT At_ij, TV_GI gt^ij, TV_EX the
// epilogue's B^i (3) and the DOF this point is the zip owner of (bits of a
// double), loaded with the other values in the prologue.
enum { TV_GT = 0, TV_AT = 1, TV_GI = 2, TV_EX = 3 };
// first x-/y-derivatives of the staged field for the mixed second derivatives
// (D_xy = D1_y D1_x, D_xz = D1_z D1_x, D_yz = D1_z D1_y), stored at the patch
// index c = x + 13y + 169z minus an offset so thread reads stay conflict-free
constexpr int TX_OFF = 3, TX_N = 2191;    // x in 3..9, y, z in 0..12
constexpr int TY_OFF = 42, TY_N = 2113;   // x, y in 3..9, z in 0..12
constexpr int T_N = 2 * STAGE_DBL;        // Tx + Ty, or two light-field stage halves
static_assert(TX_N + TY_N <= T_N, "Tx/Ty fit the two pair halves");
constexpr size_t SMEM_BYTES = size_t(NSLOT) * NPP * 8 + size_t(2) * STAGE_DBL * 8 +
                              size_t(T_N) * 8 + 16 + 16 + size_t(RT) * 4 + size_t(3) * RT * 2 + 16;

// Tensor memory as per-thread storage (tcgen05.ld / tcgen05.st, 32x32b shape:
// each thread moves 32-bit columns of its own TMEM lane).  Warp w reaches lanes
// 32 (w % 4) .. + 31 only, so the 11 warps share the 4 lane quarters and take
// column blocks of TM_WCOLS by w / 4 (3 x 48 = 144 of TM_COLS allocated; the
// radiative-boundary instantiation adds 4 blocks: 3 x 96 of 512).
// A double is two columns (low word first).  Loads complete at tcgen05.wait::ld
// (its register operands tie the loaded values to the wait).
constexpr int TM_COLS = 256, TM_WCOLS = 48;
constexpr int TM_COLS_SOMM = 512, TM_WCOLS_SOMM = 96;
// (SOMM) the radiative right-hand side of field f at a point on a domain face:
// block TV_SOMM + f / 6, parked per field stage for the epilogue
constexpr int TV_SOMM = 4;
__device__ __forceinline__ void tm_ld6(uint32_t ta, double* v) {
  uint32_t r[12];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                 "=r"(r[6]), "=r"(r[7])
               : "r"(ta));
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11])
               : "r"(ta + 8));
  asm volatile("tcgen05.wait::ld.sync.aligned;"
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]),
                 "+r"(r[6]), "+r"(r[7]), "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11])
               :
               : "memory");
#pragma unroll
  for (int i = 0; i < 6; ++i) v[i] = __hiloint2double(int(r[2 * i + 1]), int(r[2 * i]));
}
__device__ __forceinline__ void tm_st6(uint32_t ta, const double* v) {
  uint32_t r[12];
#pragma unroll
  for (int i = 0; i < 6; ++i) {
    r[2 * i] = uint32_t(__double2loint(v[i]));
    r[2 * i + 1] = uint32_t(__double2hiint(v[i]));
  }
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"r"(ta),
               "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7])
               : "memory");
  asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};" ::"r"(ta + 8),
               "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11])
               : "memory");
}
// one double (two columns)
__device__ __forceinline__ void tm_st1(uint32_t ta, double v) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" ::"r"(ta),
               "r"(uint32_t(__double2loint(v))), "r"(uint32_t(__double2hiint(v)))
               : "memory");
}
__device__ __forceinline__ void tm_st_wait() {
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// thread -> interior point map (filled by upload_rhs_tables): every warp holds
// at most two points per residue of their stage-buffer index mod 16, so its
// 8-byte stencil loads hit each of the 16 bank pairs at most twice (2
// wavefronts, conflict-free); shifted stencil taps only rotate the residues.
// (global memory, not __constant__: every thread reads a different entry)
__device__ int16_t g_perm[RT];
#ifdef DGR_RHS_TIMING
__device__ long long g_stage_cycles[NF + 2];
#endif

// Lines of the cooperative D1 pass (register pencils): threads < N_TXL take
// the x-lines of Tx (at the 133 (y, z) rows of the cross-shaped region: z in
// 3..9 with all y, or y in 3..9 with z in {0,1,2,10,11,12}), the next N_TYL the
// y-lines of Ty (x in 3..9, all z).  g_d1b[tid] is the line's first patch
// index b, assigned on the host so that the lanes of every half-warp start in
// distinct 8-byte bank pairs (b mod 16): each line's 13 loads and 7 stores are
// then conflict-free (filled by upload_rhs_tables; -1: no line)
constexpr int N_TXL = 13 * 7 + 7 * 6, N_TYL = 7 * 13;
static_assert(N_TXL + N_TYL <= RT, "one pencil per thread");
__device__ int16_t g_d1b[RT];

// the D1 pass of the staged field s: Tx = D1_x s, Ty = D1_y s (raw numerators)
// on the region the mixed stencils read (one 13-point line per thread, 20
// shared-memory accesses per 7 values)
__device__ __forceinline__ void d1_pass(const double* __restrict__ s, double* __restrict__ Tx,
                                        double* __restrict__ Ty, int tid, const int16_t* tab_d1b) {
  if (tid >= N_TXL + N_TYL) return;
  const int b = tab_d1b[tid];
  double v[13];
  if (tid < N_TXL) {
#pragma unroll
    for (int k = 0; k < 13; ++k) v[k] = s[b + k];
#pragma unroll
    for (int x = 3; x <= 9; ++x)
      Tx[b + x - TX_OFF] = (v[x + 1] - v[x - 1]) * 45.0 - (v[x + 2] - v[x - 2]) * 9.0 +
                           (v[x + 3] - v[x - 3]);
  } else {
#pragma unroll
    for (int k = 0; k < 13; ++k) v[k] = s[b + 13 * k];
#pragma unroll
    for (int y = 3; y <= 9; ++y)
      Ty[b + 13 * y - TY_OFF] = (v[y + 1] - v[y - 1]) * 45.0 - (v[y + 2] - v[y - 2]) * 9.0 +
                                (v[y + 3] - v[y - 3]);
  }
}

// field processing order: the metric gt_ij (skipped after the pre-pass), then
// the other fields with second derivatives (chi, alpha, beta^i: "heavy"),
// then the first-derivative-only ("light") fields Gt^i, K, At_ij, B^i
__constant__ int c_order[NF] = {12, 13, 14, 15, 16, 17, 1, 0, 6, 7, 8, 3,
                                4,  5,  2,  18, 19, 20, 21, 22, 23, 9, 10, 11};
__constant__ int c_order_pre[NF - 6] = {1, 0, 6, 7, 8, 3, 4, 5, 2, 18, 19, 20, 21, 22, 23, 9, 10, 11};
// fused path: the same order in stages of one or two fields — the light
// fields after the first go in pairs, the pair's second field staged in the
// Tx/Ty region (free once the last heavy stage's D1 pass is done: the first
// light stage is single, so a pair's gather, issued two stages ahead, never
// lands while a heavy stage still uses Tx/Ty).  Same per-point arithmetic in
// the same order as single stages (bit-identical to the two-pass path).
constexpr int NST_FULL = 18, NST_PRE = 12;
__constant__ int2 c_stg[NST_FULL] = {{12, -1}, {13, -1}, {14, -1}, {15, -1}, {16, -1}, {17, -1},
                                     {1, -1},  {0, -1},  {6, -1},  {7, -1},  {8, -1},  {3, -1},
                                     {4, 5},   {2, 18},  {19, 20}, {21, 22}, {23, 9},  {10, 11}};
__constant__ int2 c_stg_pre[NST_PRE] = {{1, -1},  {0, -1},  {6, -1},  {7, -1},
                                        {8, -1},  {3, -1},  {4, 5},   {2, 18},
                                        {19, 20}, {21, 22}, {23, 9},  {10, 11}};

__device__ __forceinline__ int sidx(int i, int j) {
  // (0,0)0 (0,1)1 (0,2)2 (1,1)3 (1,2)4 (2,2)5
  return i <= j ? (i == 0 ? j : (i == 1 ? 2 + j : 5)) : (j == 0 ? i : (j == 1 ? 2 + i : 5));
}

// runtime-selected entries with compile-time array indices (a dynamically
// indexed local array would live in local memory, i.e. in the L1 the gathers
// need); products of selected entries are rounded explicitly (__dmul_rn /
// __fma_rn) where they are used, so every kernel instantiation contracts them
// the same way (fused == two-pass bit for bit)
__device__ __forceinline__ double sel3(int k, double a, double b, double c) {
  return k == 0 ? a : (k == 1 ? b : c);
}
// X_{k i} of a symmetric 3x3 matrix in sidx storage, k runtime, i compile-time
__device__ __forceinline__ double row3(const double* X, int k, int i) {
  return sel3(k, X[sidx(0, i)], X[sidx(1, i)], X[sidx(2, i)]);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, int count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
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

// 8-byte asynchronous global->shared copy of (idx < ds ? uf : af)[idx] (the
// fused unzip's gather: a DOF of the state or an interpolation slot); the
// address arithmetic stays inside the asm so the compiler cannot rematerialise
// the field bases per copy
__device__ __forceinline__ void cp_async8(uint32_t dst, const double* uf, const double* af,
                                          int32_t idx, int32_t ds) {
  asm volatile(
      "{\n .reg .u64 a;\n .reg .pred q;\n setp.lt.s32 q, %3, %4;\n"
      " selp.b64 a, %1, %2, q;\n mad.wide.s32 a, %3, 8, a;\n"
      " cp.async.ca.shared.global [%0], [a], 8;\n}\n" ::"r"(dst),
      "l"(uf), "l"(af), "r"(idx), "r"(ds)
      : "memory");
}
// 8-byte asynchronous global->shared copy of *src
__device__ __forceinline__ void cp_async8u(uint32_t dst, const double* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() {
  asm volatile("cp.async.commit_group;" ::: "memory");
}
__device__ __forceinline__ void cp_async_wait1() {
  asm volatile("cp.async.wait_group 1;" ::: "memory");
}

// extrapolation rows l_m(-(t+1)), t = 0..2 (reading R12; host-computed, api.cu)
__constant__ double c_rWEXT[3 * 7];
constexpr int GJ = (NPATCH + RT - 1) / RT;   // gather points per thread (7)
constexpr int C_CENTRE = 6 + 13 * 6 + 169 * 6;   // patch centre (threads without a point)
#ifndef DGR_RKB
#define DGR_RKB 8   // (A/B, profiles/r3_experiments: 4 / 6 / 8 / 12 -> 27.60 / 27.32 / 27.25 / 27.33 ms per C3 step)
#endif
constexpr int RKB = DGR_RKB;   // fields per batch of the fused RK4 update's loads
static_assert(NF % RKB == 0, "RKB divides 24");

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

// centred 7-point stencils along one axis (stride st) at patch index c
struct Line {
  double d1, d2, ko;
};
__device__ __forceinline__ Line line_ops(const double* __restrict__ s, int c, int st) {
  const double u0 = s[c];
  const double a1 = s[c + st], b1 = s[c - st];
  const double a2 = s[c + 2 * st], b2 = s[c - 2 * st];
  const double a3 = s[c + 3 * st], b3 = s[c - 3 * st];
  Line l;
  l.d1 = (a1 - b1) * 45.0 - (a2 - b2) * 9.0 + (a3 - b3);                        // x 1/(60h)
  const double s1 = a1 + b1, s2 = a2 + b2, s3 = a3 + b3;
  l.d2 = 2.0 * s3 - 27.0 * s2 + 270.0 * s1 - 490.0 * u0;                         // x 1/(180h^2)
  l.ko = s3 - 6.0 * s2 + 15.0 * s1 - 20.0 * u0;                                  // x sigma/(64h)
  return l;
}

// Radiative condition (reading R29): d_t f = -(x^i/r) d_i f - (f - f_inf)/r at
// the domain-face node q of octant oi (x the physical coordinates), from the
// point's scaled first derivatives d1 (as derivs computes them) and value fv
__device__ __forceinline__ double somm_rhs(const DevMesh& m, int4 oi, int q, const double* d1,
                                           double fv, int f) {
  const int sd = 1 << (m.D - oi.w);
  const double unit = m.width / (6.0 * double(int64_t(1) << m.D));
  const int nd[3] = {q % 7, (q / 7) % 7, q / 49}, an[3] = {oi.x, oi.y, oi.z};
  double xr = 0.0, r2 = 0.0;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    const double x = m.xmin[a] + double(6 * int64_t(an[a]) + int64_t(nd[a]) * sd) * unit;
    xr = __fma_rn(x, d1[a], xr);
    r2 = __fma_rn(x, x, r2);
  }
  const double finf = (f <= 1 || f == 12 || f == 15 || f == 17) ? 1.0 : 0.0;
  const double ir = 1.0 / sqrt(r2);
  return __fma_rn(-xr, ir, -(fv - finf) * ir);
}

// the radiative value of staged field f at the point (patch index c0 of s),
// stored in TMEM at column address ta (first derivatives as derivs computes them)
__device__ __forceinline__ void somm_park(const DevMesh& m, int4 oi, int q, const double* s, int c0,
                                          double ih, int f, uint32_t ta) {
  const double f1 = ih * (1.0 / 60.0);
  const double d1[3] = {line_ops(s, c0, 1).d1 * f1, line_ops(s, c0, 13).d1 * f1,
                        line_ops(s, c0, 169).d1 * f1};
  tm_st1(ta, somm_rhs(m, oi, q, d1, s[c0], f));
}

// D1_b(D1_a u) * (60h)^2
__device__ __forceinline__ double mixed(const double* __restrict__ s, int c, int sa, int sb) {
  double r[7];
#pragma unroll
  for (int b = -3; b <= 3; ++b) {
    if (b == 0) continue;
    const int cb = c + b * sb;
    r[b + 3] = (s[cb + sa] - s[cb - sa]) * 45.0 - (s[cb + 2 * sa] - s[cb - 2 * sa]) * 9.0 +
               (s[cb + 3 * sa] - s[cb - 3 * sa]);
  }
  return (r[4] - r[2]) * 45.0 - (r[5] - r[1]) * 9.0 + (r[6] - r[0]);
}

struct Derivs {
  double d1[3];
  double dd[6];  // symmetric second derivatives (only if second)
  double ko;     // sum of the 3 KO terms, already scaled
};

template <bool SECOND>
__device__ __forceinline__ Derivs derivs(const double* __restrict__ s, int c, double ih,
                                         double ko_scale) {
  Derivs d;
  const Line lx = line_ops(s, c, 1), ly = line_ops(s, c, 13), lz = line_ops(s, c, 169);
  const double f1 = ih * (1.0 / 60.0);
  d.d1[0] = lx.d1 * f1;
  d.d1[1] = ly.d1 * f1;
  d.d1[2] = lz.d1 * f1;
  d.ko = __dmul_rn(lx.ko + ly.ko + lz.ko, ko_scale);
  if (SECOND) {
    const double f2 = ih * ih * (1.0 / 180.0);
    const double fm = ih * ih * (1.0 / 3600.0);
    d.dd[0] = lx.d2 * f2;
    d.dd[3] = ly.d2 * f2;
    d.dd[5] = lz.d2 * f2;
    d.dd[1] = mixed(s, c, 1, 13) * fm;
    d.dd[2] = mixed(s, c, 1, 169) * fm;
    d.dd[4] = mixed(s, c, 13, 169) * fm;
  }
  return d;
}

// (callers add the KO term with __dadd_rn and derivs* round it with __dmul_rn,
// so no kernel instantiation fuses the two: fused == two-pass bit for bit)
// advective derivative beta^k d_k f at patch index c: reading R9, the centred
// D1 (d1 = its values); with upw (dgr_params.upwind, reading R9u) the 4th-order
// lopsided stencil (-3 f_-1 - 10 f_0 + 18 f_1 - 6 f_2 + f_3) / (12 h) shifted
// towards +k where beta^k >= 0 and its mirror image where beta^k < 0
template <bool UPW>
__device__ __forceinline__ double advect(const double* __restrict__ s, int c, const double* beta,
                                         const double* d1, double ih) {
  if (!UPW) return beta[0] * d1[0] + beta[1] * d1[1] + beta[2] * d1[2];
  // (rounding pinned by explicit fma / mul: the sign selects would otherwise let
  // different kernel instantiations contract differently)
  double a = 0.0;
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    const int st = k == 0 ? 1 : (k == 1 ? 13 : 169);
    const int q = beta[k] >= 0.0 ? st : -st;
    const double e =
        __fma_rn(-3.0, s[c - q],
                 __fma_rn(-10.0, s[c], __fma_rn(18.0, s[c + q], __fma_rn(-6.0, s[c + 2 * q], s[c + 3 * q]))));
    a = __fma_rn(beta[k], __dmul_rn(beta[k] >= 0.0 ? e : -e, ih * (1.0 / 12.0)), a);
  }
  return a;
}

// D1 of a precomputed D1 field (raw numerators), at patch index c
__device__ __forceinline__ double d1_of(const double* __restrict__ T, int c, int st) {
  return (T[c + st] - T[c - st]) * 45.0 - (T[c + 2 * st] - T[c - 2 * st]) * 9.0 +
         (T[c + 3 * st] - T[c - 3 * st]);
}

// first, pure second and mixed derivatives + KO; the mixed ones from the
// cooperative Tx = D1_x u and Ty = D1_y u fields (same D1 o D1 stencil, R10)
__device__ __forceinline__ Derivs derivs2(const double* __restrict__ s,
                                          const double* __restrict__ Tx,
                                          const double* __restrict__ Ty, int c, double ih,
                                          double ko_scale) {
  Derivs d;
  const Line lx = line_ops(s, c, 1), ly = line_ops(s, c, 13), lz = line_ops(s, c, 169);
  const double f1 = ih * (1.0 / 60.0);
  d.d1[0] = lx.d1 * f1;
  d.d1[1] = ly.d1 * f1;
  d.d1[2] = lz.d1 * f1;
  d.ko = __dmul_rn(lx.ko + ly.ko + lz.ko, ko_scale);
  const double f2 = ih * ih * (1.0 / 180.0);
  const double fm = ih * ih * (1.0 / 3600.0);
  d.dd[0] = lx.d2 * f2;
  d.dd[3] = ly.d2 * f2;
  d.dd[5] = lz.d2 * f2;
  d.dd[1] = d1_of(Tx, c - TX_OFF, 13) * fm;
  d.dd[2] = d1_of(Tx, c - TX_OFF, 169) * fm;
  d.dd[4] = d1_of(Ty, c - TY_OFF, 169) * fm;
  return d;
}

// stores of results read back only by a later kernel (the pre-pass rows, the
// DOF-ordered RHS): DGR_STREAM_STORES marks them evict-first so they do not
// push the gather sources out of L2
__device__ __forceinline__ void st_out(double* p, double v) {
#ifdef DGR_STREAM_STORES
  __stcs(p, v);
#else
  *p = v;
#endif
}

// TF_ONCE (default): the trace-free projection of eq (6)'s chi[..]^TF terms is
// linear, so it is applied once in the epilogue (sum c X - gt/3 sum c tr X)
// instead of in each of the six stages that contribute (C3 RHS 7.12 -> 7.03 ms);
// -DDGR_TF_PER_STAGE restores the per-stage projection (experiment builds)
#ifdef DGR_TF_PER_STAGE
constexpr bool TF_ONCE = false;
#else
constexpr bool TF_ONCE = true;
#endif

// trace with the inverse metric: gt^ij X_ij (symmetric storage)
__device__ __forceinline__ double trace6(const double* gi, const double* X) {
  return gi[0] * X[0] + gi[3] * X[3] + gi[5] * X[5] +
         2.0 * (gi[1] * X[1] + gi[2] * X[2] + gi[4] * X[4]);
}

// v^i = At^ij w_j with At^ij = gt^ik gt^jl At_kl, contracted vector-first
// (w^l = gt^lj w_j, y_k = At_kl w^l, v^i = gt^ik y_k: 27 FMAs)
__device__ __forceinline__ void at_up_w(const double* gi, const double* At, const double* w,
                                        double* v) {
  double wu[3], y[3];
#pragma unroll
  for (int l = 0; l < 3; ++l)
    wu[l] = gi[sidx(l, 0)] * w[0] + gi[sidx(l, 1)] * w[1] + gi[sidx(l, 2)] * w[2];
#pragma unroll
  for (int k = 0; k < 3; ++k)
    y[k] = At[sidx(k, 0)] * wu[0] + At[sidx(k, 1)] * wu[1] + At[sidx(k, 2)] * wu[2];
#pragma unroll
  for (int i = 0; i < 3; ++i)
    v[i] = gi[sidx(i, 0)] * y[0] + gi[sidx(i, 1)] * y[1] + gi[sidx(i, 2)] * y[2];
}

// the thread -> point map (g_perm) and the D1-pass line table (g_d1b), host side
inline void build_rhs_tables(int16_t* perm, int16_t* d1b) {
  std::vector<int> bucket[16];
  for (int p = 0; p < NPT; ++p) {
    const int c = (p % 7 + 3) + 13 * ((p / 7) % 7 + 3) + 169 * (p / 49 + 3);
    bucket[c % 16].push_back(p);
  }
  size_t next[16] = {0};
  for (int t = 0; t < RT; ++t) perm[t] = -1;
  for (int w = 0; w < RT / 32; ++w)
    for (int lane = 0; lane < 32; ++lane) {
      const int r = lane % 16;
      if (next[r] < bucket[r].size()) perm[w * 32 + lane] = int16_t(bucket[r][next[r]++]);
    }
  // D1-pass lines: per kind, fill each half-warp with lines of distinct b mod 16
  // (greedy, the most frequent residues first)
  for (int t = 0; t < RT; ++t) d1b[t] = -1;
  std::vector<int> lx, ly;
  for (int z = 3; z <= 9; ++z)
    for (int y = 0; y < 13; ++y) lx.push_back(13 * y + 169 * z);
  for (int z = 0; z < 13; ++z)
    if (z < 3 || z > 9)
      for (int y = 3; y <= 9; ++y) lx.push_back(13 * y + 169 * z);
  for (int z = 0; z < 13; ++z)
    for (int x = 3; x <= 9; ++x) ly.push_back(x + 169 * z);
  auto assign = [&](std::vector<int>& lines, int t0, int t1) {
    std::vector<std::vector<int>> byres(16);
    for (int b : lines) byres[b % 16].push_back(b);
    for (int h = t0; h < t1;) {
      const int he = std::min(t1, (h / 16 + 1) * 16);   // the part of this half-warp in [t0, t1)
      bool used[16] = {false};
      for (int t = h; t < he; ++t) {
        int best = -1;
        for (int r = 0; r < 16; ++r)
          if (!used[r] && !byres[r].empty() && (best < 0 || byres[r].size() > byres[best].size()))
            best = r;
        if (best < 0)   // every residue left is taken in this half-warp: any line
          for (int r = 0; r < 16; ++r)
            if (!byres[r].empty() && (best < 0 || byres[r].size() > byres[best].size())) best = r;
        used[best] = true;
        d1b[t] = int16_t(byres[best].back());
        byres[best].pop_back();
      }
      h = he;
    }
  };
  assign(lx, 0, N_TXL);
  assign(ly, N_TXL, N_TXL + N_TYL);
}

// this translation unit's copies of the tables
inline void upload_tables_here(const double* wext) {
  cudaMemcpyToSymbol(c_rWEXT, wext, sizeof(double) * 21);
  int16_t perm[RT], d1b[RT];
  build_rhs_tables(perm, d1b);
  cudaMemcpyToSymbol(g_perm, perm, sizeof(perm));
  cudaMemcpyToSymbol(g_d1b, d1b, sizeof(d1b));
}

}  // namespace
}  // namespace dgr
