// Fused BSSN RHS kernel: 6th-order derivatives + KO + the 24-field algebra
// (§III-A eqs 1-19, §IV-B), fp64, sm_100a.
//
// Design: one persistent CTA per SM, one thread per interior
// point (343 of 352 threads).  The field patches stream through shared memory
// one (or, for first-derivative-only fields, two) at a time: gathered from
// the state and the interpolation slots with 8-byte cp.async (the fused
// unzip, default) or bulk-copied from a patch buffer (cp.async.bulk, mbarrier
// completion); double buffered across octant boundaries.  While a field is
// resident every thread evaluates that field's derivatives at its point
// straight from shared memory and immediately consumes them in the part of
// the algebra that only needs them ("staged" evaluation, cf. the paper's
// staged+CSE), so the 210 derivatives of P:L310 are never stored.
// State that survives between fields: the point's read-only values (gt_ij,
// At_ij, gt^ij, B^i, its zip-owner DOF) in tensor memory, one TMEM lane per
// thread (tcgen05.ld / tcgen05.st); the accumulators of the 21 vector/tensor
// outputs and the Christoffel scratch in shared-memory slots [slot][thread].
// The epilogue zips by its store and, in dgr_rk4_step, applies the RK4 stage
// update.  The metric pre-pass (k_gt_pre, below) takes the gt_ij fields.
// Field order:
//   gt_ij (6) -> [Christoffel block] -> chi -> alpha -> beta^i (3) -> Gt^i (3)
//   -> K -> At_ij (6) -> B^i (3)
// Readings: R1-R8, R13; chi in divisions is max(chi, chi_floor).
// Two algebraically exact simplifications versus the oracle's literal form:
// the gt_ij-proportional part of R^chi_ij (eq 19) is dropped because the
// trace-free projection in eq (6) annihilates it, and Gt_ijk (lowered) is the
// first-kind symbol C_ijk itself (gt_il gt^lm C_mjk = C_ijk).
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

}  // namespace

// FUSED = false: `patches` is the 13^3 patch buffer [24][n_owned][PATCH_PITCH]
// (bulk copies).  FUSED = true: `patches` is the state u and every patch is
// gathered straight from u and the interpolation slots through m.gmap with
// 8-byte cp.async (the unzip fused into the RHS), and
// points outside a non-periodic domain are extrapolated in shared memory with
// the same arithmetic as k_unzip.
// SOMM: radiative outer boundary (reading R29) compiled in (a separate
// instantiation, so the default path carries none of its registers).
// UPW: lopsided advective derivatives (reading R9u, dgr_params.upwind) compiled in
template <bool FUSED, bool SOMM, bool PRE, bool UPW>
__global__ void __launch_bounds__(RT, 1)
    k_rhs(DevMesh m, const double* __restrict__ patches, double* __restrict__ rhs_oct,
          RhsParams prm, int first, int count, const double* __restrict__ pre,
          double* __restrict__ rhs_dof) {
  // PRE: the gt_ij stages were done by k_gt_pre (its 30 values per point are
  // read in the prologue); the stream holds the 18 other fields
  constexpr int NS = PRE ? NF - 6 : NF;
  const int* ORD = PRE ? c_order_pre : c_order;
  // stages: FUSED in one- or two-field stages (c_stg*), else one field each
  constexpr int NST = FUSED ? (PRE ? NST_PRE : NST_FULL) : NS;
  const int2* STG = PRE ? c_stg_pre : c_stg;
  auto stA = [&](int k) { return FUSED ? STG[k].x : ORD[k]; };
  auto stB = [&](int k) { return FUSED ? STG[k].y : -1; };
  extern __shared__ __align__(128) double smem[];
  double* slots = smem;                           // [NSLOT][NPP]
  double* stage = smem + NSLOT * NPP;             // [2][STAGE_DBL]
  double* Tx = stage + 2 * STAGE_DBL;             // [TX_N] (T region: [T_N])
  double* Ty = Tx + TX_N;                         // [TY_N]
  uint64_t* bars = reinterpret_cast<uint64_t*>(Tx + T_N);
  // FUSED: the octant-to-come's anchor (16 B) and each thread's o2s index of
  // its point in it, copied asynchronously two stages before its prologue
  int4* sm_oi = reinterpret_cast<int4*>(bars + 2);
  int32_t* tab_cv = reinterpret_cast<int32_t*>(sm_oi + 1);
  // this thread's point: patch index c0 (-1: no point) and interior index p, kept
  // in shared memory and re-read where needed (cheaper than a register spill)
  int16_t* tab_c0 = reinterpret_cast<int16_t*>(tab_cv + RT);
  int16_t* tab_p = tab_c0 + RT;
  int16_t* tab_d1b = tab_p + RT;                                  // D1-pass line (g_d1b)
  uint32_t* tm_base = reinterpret_cast<uint32_t*>(tab_d1b + RT);  // TMEM allocation address

  const int tid = threadIdx.x;
  {
    const int pp = g_perm[tid];
    const int q = pp >= 0 ? pp : 0;
    tab_c0[tid] = pp >= 0 ? int16_t((q % 7 + 3) + 13 * ((q / 7) % 7 + 3) + 169 * (q / 49 + 3)) : -1;
    tab_p[tid] = int16_t(q);
    tab_d1b[tid] = g_d1b[tid];
  }
  const int64_t no = m.n_owned;
  const int64_t fstride = FUSED ? m.dof_stride : no * PATCH_PITCH;
  const int32_t ds = int32_t(m.dof_stride);
  int gidx[GJ];   // FUSED: SRC index of patch points tid + RT*j of the current octant
  int gdst[GJ];   // FUSED: patch point each of this thread's copies fills
  auto load_gidx = [&](int oct) {
    // entries sorted by source (m.gmap_s): a warp's copies read few lines
    const int32_t* gm = m.gmap_s + int64_t(oct) * GM_PITCH;
    const int16_t* gd = m.gdst + int64_t(oct) * GM_PITCH;
#pragma unroll
    for (int j = 0; j < GJ; ++j) {
      const int pt = tid + RT * j;
      // (extrapolated points, -1, copy a dummy value and are overwritten later)
      gidx[j] = pt < NPATCH ? max(__ldg(gm + pt), 0) : -1;
      gdst[j] = pt < NPATCH ? int(__ldg(gd + pt)) : 0;
    }
  };
  auto gather = [&](double* dst, int f) {
    // only the points the field's stencils read: the cross region for the
    // first-derivative-only fields, the three slabs for the others
    const bool sec = f <= 1 || (f >= 6 && f <= 8) || (f >= 12 && f <= 17);
    const int n = sec ? G_SLABS : G_CROSS;
    const uint32_t d0 = smem_u32(dst);
    const double* uf = patches + f * fstride;
    const double* af = m.aux + f * m.aux_stride - m.dof_stride;
#pragma unroll
    for (int j = 0; j < GJ; ++j)
      if (tid + RT * j < n) cp_async8(d0 + 8 * gdst[j], uf, af, gidx[j], ds);
  };
  // FUSED: stage k's field(s) into stage buffer b (and T-region half b), one
  // cp.async group per stage
  // (oct_next >= 0: also the next octant's anchor and o2s index, which land
  // with this group, before that octant's prologue)
  auto gather_stage = [&](int b, int k, int oct_next = -1) {
    gather(stage + b * STAGE_DBL, stA(k));
    if (stB(k) >= 0) gather(Tx + b * STAGE_DBL, stB(k));
    if (oct_next >= 0) {
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(tab_cv + tid)),
                   "l"(m.o2s + int64_t(oct_next) * NPT + max(int(tab_p[tid]), 0))
                   : "memory");
      if (tid == 0)
        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(smem_u32(sm_oi)),
                     "l"(m.oct + oct_next)
                     : "memory");
    }
    cp_async_commit();
  };
  // FUSED: the value of field f at element node (e, p), through o2s
  auto node_value = [&](int f, int oct, int node) {
    const int32_t x = __ldg(m.o2s + int64_t(oct) * NPT + node);
    return x < ds ? __ldg(patches + f * fstride + x) : __ldg(m.aux + f * m.aux_stride + (x - ds));
  };
#define SL(slot) slots[(slot) * NPP + tid]
  auto prefetch_l2 = [&](const double* src) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src),
                 "r"(uint32_t(STAGE_DBL * 8))
                 : "memory");
  };

  // Persistent CTAs: octants e = blockIdx.x, +gridDim.x, ...  The field stream
  // (double-buffered bulk copies, mbarrier phase = global stage count) runs
  // on across octant boundaries, and the next octant's 24 field patches are
  // prefetched into L2 one octant ahead.
  // (octant list m.olist[first, first + count): interior octants before the
  // ones that wait for ghost values, api.cu)
  const int32_t* ol = m.olist + first;
  int li = blockIdx.x;
  if (li >= count) return;
  int e = ol[li];
  if (tid == 0) {
    mbar_init(&bars[0], 1);
    mbar_init(&bars[1], 1);
  }
  if (tid < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tm_base)),
                 "n"(SOMM ? TM_COLS_SOMM : TM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (FUSED) {   // the first octant's anchor and o2s index (later ones arrive by cp.async)
    tab_cv[tid] = __ldg(m.o2s + int64_t(e) * NPT + max(int(tab_p[tid]), 0));
    if (tid == 0) *sm_oi = m.oct[e];
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  // this thread's TMEM address (lane quarter of its warp, column block)
  const uint32_t tma = *tm_base + (uint32_t(32 * ((tid >> 5) & 3)) << 16) +
                       (SOMM ? TM_WCOLS_SOMM : TM_WCOLS) * (tid >> 7);
#define VALS_LD(w, v) tm_ld6(tma + 12 * (w), v)
#define VALS_ST(w, v) tm_st6(tma + 12 * (w), v)

  if (FUSED) {
    load_gidx(e);
    gather_stage(0, 0);
    gather_stage(1, 1);
  } else if (tid == 0) {
    const double* pb = patches + int64_t(e) * PATCH_PITCH;
    bulk_load(stage, pb + ORD[0] * fstride, STAGE_DBL * 8, &bars[0]);
    bulk_load(stage + STAGE_DBL, pb + ORD[1] * fstride, STAGE_DBL * 8, &bars[1]);
  } else if (tid < NS - 1) {
    prefetch_l2(patches + int64_t(e) * PATCH_PITCH + ORD[tid + 1] * fstride);
  }
  uint32_t g = 0;   // global stage counter of this CTA
  for (; li < count; li += gridDim.x) {
  e = ol[li];
  const int en = li + int(gridDim.x) < count ? ol[li + gridDim.x] : -1;   // next octant of this CTA
  const double* pbase = patches + int64_t(e) * (FUSED ? NPT : PATCH_PITCH);
  // (threads without a point — 9 of 352 — run the same code on the patch
  // centre / element node 0 and store nothing: TMEM accesses are warp-wide)
  const bool active = tab_c0[tid] >= 0;
  // the point's own values: patch index c0 of the staged patches, or (FUSED)
  // element node p of u / a hanging-node slot through o2s
  const int cv = FUSED ? tab_cv[tid]
                       : (active ? int(tab_c0[tid]) : C_CENTRE);
  auto own = [&](int f) -> double {
    if (!FUSED) return __ldg(pbase + f * fstride + cv);
    return cv < ds ? __ldg(patches + f * fstride + cv) : __ldg(m.aux + f * m.aux_stride + (cv - ds));
  };

  const int4 oi = FUSED ? *sm_oi : m.oct[e];
  // FUSED: which faces of this octant lie on a non-periodic domain boundary
  // (bit a: low face along axis a outside the domain, bit 3 + a: high face)
  int omask = 0;
  if (FUSED && !m.periodic) {
    const int nside = 1 << m.D, sd = 1 << (m.D - oi.w);
    omask = (oi.x == 0) | ((oi.y == 0) << 1) | ((oi.z == 0) << 2) | ((oi.x + sd == nside) << 3) |
            ((oi.y + sd == nside) << 4) | ((oi.z + sd == nside) << 5);
  }
  const bool bnd = omask != 0;
  if (FUSED && en >= 0 && tid == 32) {   // next octant's gather rows (gmap_s, gdst) into L2
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(m.gmap_s + int64_t(en) * GM_PITCH),
                 "r"(uint32_t(GM_PITCH * 4))
                 : "memory");
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(m.gdst + int64_t(en) * GM_PITCH),
                 "r"(uint32_t(GM_PITCH * 2))
                 : "memory");
  }
  const double ih = (6.0 * double(int64_t(1) << oi.w)) / m.width;   // 1/h
  const double ko_scale = prm.ko_sigma * ih * (1.0 / 64.0);
  // Sommerfeld (reading R29): this point is a node on a face of the domain
  bool bpt = false;
  if (SOMM && tab_c0[tid] >= 0) {
    const int q = tab_p[tid], nx = q % 7, ny = (q / 7) % 7, nz = q / 49;
    const int nside = 1 << m.D, sd = 1 << (m.D - oi.w);
    bpt = (nx == 0 && oi.x == 0) || (ny == 0 && oi.y == 0) || (nz == 0 && oi.z == 0) ||
          (nx == 6 && oi.x + sd == nside) || (ny == 6 && oi.y + sd == nside) ||
          (nz == 6 && oi.z + sd == nside);
  }
  // (SOMM) some point of this warp is on a domain face: warp-uniform, so the
  // warp-wide TMEM stores and loads of the radiative values run only there
  const bool bwarp = SOMM && __any_sync(0xffffffffu, bpt);

  // ---- values at the point (patch interior) -------------------------------
  if (PRE) {
    // metric pre-pass results -> d gt (S0), gt^lm d_lm gt (A_AT), adv + KO of gt
    // (A_GAM) slots, asynchronously, in flight while the values are read
    // (pre rows are indexed by thread, [c][n_owned][RT]: coalesced)
    const double* pr = pre + int64_t(e) * RT + tid;
    const int64_t pstr = no * RT;
#pragma unroll
    for (int i = 0; i < 18; ++i) cp_async8u(smem_u32(&SL(S0 + i)), pr + i * pstr);
#pragma unroll
    for (int q = 0; q < 6; ++q) {
      cp_async8u(smem_u32(&SL(A_AT + q)), pr + (18 + q) * pstr);
      cp_async8u(smem_u32(&SL(A_GAM + q)), pr + (24 + q) * pstr);
    }
    cp_async_commit();
  }
  double alpha, chi, Kv, beta[3];
  {
    alpha = own(0);
    chi = own(1);
    Kv = own(2);
#pragma unroll
    for (int i = 0; i < 3; ++i) beta[i] = own(6 + i);
    double g[6], at[6];
#pragma unroll
    for (int q = 0; q < 6; ++q) {
      g[q] = own(12 + q);
      at[q] = own(18 + q);
    }
    VALS_ST(TV_GT, g);
    VALS_ST(TV_AT, at);
    {
      // the epilogue's B^i and zip-owner DOF, in flight with the values above
      const int dz = rhs_dof && active ? __ldg(m.own + int64_t(e) * NPT + max(int(tab_p[tid]), 0)) : -1;
      const double ex[6] = {own(9), own(10), own(11), __hiloint2double(0, dz), 0.0, 0.0};
      VALS_ST(TV_EX, ex);
    }
    // inverse metric by adjugate / determinant
    const double a00 = g[3] * g[5] - g[4] * g[4];
    const double a01 = g[2] * g[4] - g[1] * g[5];
    const double a02 = g[1] * g[4] - g[2] * g[3];
    const double det = g[0] * a00 + g[1] * a01 + g[2] * a02;
    const double idet = 1.0 / det;
    double gi[6];
    gi[0] = a00 * idet;
    gi[1] = a01 * idet;
    gi[2] = a02 * idet;
    gi[3] = (g[0] * g[5] - g[2] * g[2]) * idet;
    gi[4] = (g[1] * g[2] - g[0] * g[4]) * idet;
    gi[5] = (g[0] * g[3] - g[1] * g[1]) * idet;
    VALS_ST(TV_GI, gi);
    tm_st_wait();
#pragma unroll
    for (int q = 0; q < 6; ++q) SL(A_GT + q) = 0.0;     // A_GT, A_BETA
    if (!PRE) {
#pragma unroll
      for (int q = 0; q < 6; ++q) SL(A_GAM + q) = 0.0;
    }
  }
  const double chi_e = fmax(chi, prm.chi_floor);
  const double ichi = 1.0 / chi_e;
  double rA = 0.0, rC = 0.0, rK = 0.0;   // accumulators of alpha, chi, K
  double ttr = 0.0;   // (TF_ONCE) sum of c * gt^ij X_ij over the trace-free terms of eq (6)
  double dchi[3] = {0, 0, 0};

  // Christoffel block (eqs 12, 17; readings R1, R7): from d_k gt_ij (S0 slots)
  // and gt^lm d_lm gt_ij (A_AT slots) — at the last gt stage, or (PRE) right
  // after the prologue from the metric pre-pass
  auto christoffel = [&](const double* gi) {
      // ---------------- Christoffel block (eqs 12, 17; readings R1, R7)
      double gt[6], At[6];
      VALS_LD(TV_GT, gt);
      VALS_LD(TV_AT, At);
      double C[3][6];  // first kind C_k,ij = 1/2 (d_i g_kj + d_j g_ki - d_k g_ij)
#pragma unroll
      for (int k = 0; k < 3; ++k)
#pragma unroll
        for (int i = 0; i < 3; ++i)
#pragma unroll
          for (int j = i; j < 3; ++j)
            C[k][sidx(i, j)] = 0.5 * (SL(S0 + i * 6 + sidx(k, j)) + SL(S0 + j * 6 + sidx(k, i)) -
                                      SL(S0 + k * 6 + sidx(i, j)));
      double Gam[3][6];  // second kind Gt^k_ij = gt^kl C_l,ij
#pragma unroll
      for (int k = 0; k < 3; ++k)
#pragma unroll
        for (int q2 = 0; q2 < 6; ++q2)
          Gam[k][q2] = gi[sidx(k, 0)] * C[0][q2] + gi[sidx(k, 1)] * C[1][q2] +
                       gi[sidx(k, 2)] * C[2][q2];
      double cal[3];
#pragma unroll
      for (int k = 0; k < 3; ++k) cal[k] = trace6(gi, Gam[k]);
      // Rt_ij without the d Gt terms
      double Rt[6];
      // gt^lm (Gt^k_li C_j,km + Gt^k_lj C_i,km + Gt^k_im C_k,lj) with the metric
      // contracted first: Cu[a][b][c] = gt^cm C_a,bm, so each (i,j) needs 27 FMAs
      // (Gt^k_li Cu[j][k][l] + Gt^k_lj Cu[i][k][l] + Gt^k_im Cu[k][j][m])
#pragma unroll
      for (int i = 0; i < 3; ++i)
#pragma unroll
        for (int j = i; j < 3; ++j) {
          double c2 = 0.0;
#pragma unroll
          for (int k = 0; k < 3; ++k) c2 += cal[k] * (C[i][sidx(j, k)] + C[j][sidx(i, k)]);
          Rt[sidx(i, j)] = -0.5 * SL(A_AT + sidx(i, j)) + 0.5 * c2;
        }
      double Cu[3][3][3];
#pragma unroll
      for (int a = 0; a < 3; ++a)
#pragma unroll
        for (int b = 0; b < 3; ++b)
#pragma unroll
          for (int c = 0; c < 3; ++c)
            Cu[a][b][c] = gi[sidx(c, 0)] * C[a][sidx(b, 0)] + gi[sidx(c, 1)] * C[a][sidx(b, 1)] +
                          gi[sidx(c, 2)] * C[a][sidx(b, 2)];
#pragma unroll
      for (int i = 0; i < 3; ++i)
#pragma unroll
        for (int j = i; j < 3; ++j) {
          double qsum = 0.0;
#pragma unroll
          for (int k = 0; k < 3; ++k)
#pragma unroll
            for (int l = 0; l < 3; ++l)
              qsum += Gam[k][sidx(l, i)] * Cu[j][k][l] + Gam[k][sidx(l, j)] * Cu[i][k][l] +
                      Gam[k][sidx(i, l)] * Cu[k][j][l];
          Rt[sidx(i, j)] += qsum;
        }
      // At_ij = chi alpha TF(Rt)   (first write of the A_AT accumulators)
      const double trR = trace6(gi, Rt);
      const double ca = chi * alpha;
      if (TF_ONCE) {
#pragma unroll
        for (int r = 0; r < 6; ++r) SL(A_AT + r) = ca * Rt[r];
        ttr += ca * trR;
      } else {
#pragma unroll
        for (int r = 0; r < 6; ++r) SL(A_AT + r) = ca * (Rt[r] - gt[r] * trR * (1.0 / 3.0));
      }
      // At^ij = gt^ik gt^jl At_kl ; Gt^i += 2 alpha Gt^i_jk At^jk
      double Au[6];
      {
        double M[3][3];   // At_k^j = At_kl gt^lj
#pragma unroll
        for (int k = 0; k < 3; ++k)
#pragma unroll
          for (int j = 0; j < 3; ++j)
            M[k][j] = At[sidx(k, 0)] * gi[sidx(0, j)] + At[sidx(k, 1)] * gi[sidx(1, j)] +
                      At[sidx(k, 2)] * gi[sidx(2, j)];
#pragma unroll
        for (int i = 0; i < 3; ++i)
#pragma unroll
          for (int j = i; j < 3; ++j)
            Au[sidx(i, j)] = gi[sidx(i, 0)] * M[0][j] + gi[sidx(i, 1)] * M[1][j] +
                             gi[sidx(i, 2)] * M[2][j];
      }
#pragma unroll
      for (int i = 0; i < 3; ++i) SL(A_GT + i) += 2.0 * alpha * trace6(Au, Gam[i]);
      // keep Gt^k_ij and CalGt^k for the chi, alpha and beta stages
#pragma unroll
      for (int k = 0; k < 3; ++k)
#pragma unroll
        for (int q2 = 0; q2 < 6; ++q2) SL(S0 + k * 6 + q2) = Gam[k][q2];
#pragma unroll
      for (int k = 0; k < 3; ++k) SL(A_B + k) = cal[k];   // (A_B slot reused until B)
      };
#ifdef DGR_RHS_TIMING
  long long t_last = clock64();
#endif
  if (PRE) {
    // the metric pre-pass results for this point (copies issued before the
    // point's values were read), then the Christoffel block
    asm volatile("cp.async.wait_all;" ::: "memory");
    double gi[6];
    VALS_LD(TV_GI, gi);
    if (SOMM && bwarp) {
      // the gt_ij fields' radiative values (reading R29) from their pre-pass
      // first derivatives, before the Christoffel block reuses the S0 slots
      double gq[6];
      VALS_LD(TV_GT, gq);
      const int c0 = active ? int(tab_c0[tid]) : C_CENTRE;
      (void)c0;
#pragma unroll
      for (int q = 0; q < 6; ++q) {
        const double d1[3] = {SL(S0 + q), SL(S0 + 6 + q), SL(S0 + 12 + q)};
        tm_st1(tma + 2 * (6 * TV_SOMM + 12 + q), somm_rhs(m, oi, int(tab_p[tid]), d1, gq[q], 12 + q));
      }
    }
    christoffel(gi);
  }
  for (int st = 0; st < NST; ++st, ++g) {
    const int buf = g & 1;
#ifdef DGR_RHS_TIMING
    if (tid == 0) {   // per-stage cycle profile (experiment builds only)
      const long long t = clock64();
      atomicAdd(reinterpret_cast<unsigned long long*>(&g_stage_cycles[st]),
                (unsigned long long)(t - t_last));
      t_last = t;
    }
#endif
    if (FUSED) {
      cp_async_wait1();   // this thread's copies of stage st have landed
      __syncthreads();    // ... and everyone else's
      if (bnd) {
        // outer-boundary extrapolation along x, then y, then z (reading R12),
        // the arithmetic of k_unzip, in shared memory (both fields of a pair)
        for (int hb = 0; hb < (stB(st) >= 0 ? 2 : 1); ++hb) {
        double* sw = (hb ? Tx : stage) + buf * STAGE_DBL;
        for (int a = 0; a < 3; ++a) {
          const int sa = a == 0 ? 1 : (a == 1 ? 13 : 169);
          const int sb = a == 0 ? 13 : 1, sc = a == 2 ? 13 : 169;
          const int b_ax = a == 0 ? 1 : 0, c_ax = a == 2 ? 1 : 2;
          for (int side = 0; side < 2; ++side) {
            if (!((omask >> (a + 3 * side)) & 1)) continue;
            for (int idx = tid; idx < 3 * 169; idx += RT) {
              const int k3 = idx % 3, uv = idx / 3;
              const int cb = uv % 13, cc = uv / 13;
              if (b_ax > a && ((cb < 3 && ((omask >> b_ax) & 1)) || (cb > 9 && ((omask >> (3 + b_ax)) & 1))))
                continue;
              if (c_ax > a && ((cc < 3 && ((omask >> c_ax) & 1)) || (cc > 9 && ((omask >> (3 + c_ax)) & 1))))
                continue;
              const int ia = side == 0 ? k3 : 10 + k3;
              const int base = cb * sb + cc * sc;
              double acc = 0.0;
              if (side == 0) {
                const double* w = c_rWEXT + (2 - ia) * 7;
#pragma unroll
                for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], sw[base + (3 + mm) * sa], acc);
              } else {
                const double* w = c_rWEXT + (ia - 10) * 7;
#pragma unroll
                for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], sw[base + (9 - mm) * sa], acc);
              }
              sw[base + ia * sa] = acc;
            }
          }
          __syncthreads();
        }
        }
      }
    } else {
      mbar_wait(&bars[buf], (g >> 1) & 1);
    }
    const double* s = stage + buf * STAGE_DBL;
    const int f = stA(st);
    const bool second = f <= 1 || (f >= 6 && f <= 8) || (f >= 12 && f <= 17);
    if (second) {
      // cooperative first derivatives along x (and y) of the staged field on
      // the extended region the mixed stencils need (d1_pass: register
      // pencils, one conflict-free 13-point line per thread)
      d1_pass(s, Tx, Ty, tid, tab_d1b);
      __syncthreads();
    }
    // the per-point work of a first-derivative-only ("light") field f from its
    // derivatives d (s: its staged patch, which the lopsided advection reads)
    auto light_apply = [&](const double* __restrict__ s, const int f, const Derivs& d) {
      const int c0 = active ? int(tab_c0[tid]) : C_CENTRE;
      if (f >= 3 && f <= 5) {
        // ---------------- Gt^k: Ricci d Gt term, advection + KO kept apart (eq 3)
        const int kk = f - 3;
        SL(S0 + kk) = __dadd_rn(advect<UPW>(s, c0, beta, d.d1, ih), d.ko);
        double gi[6], gt[6], Rg[6];
        VALS_LD(TV_GI, gi);
        VALS_LD(TV_GT, gt);
#pragma unroll
        for (int i = 0; i < 3; ++i)
#pragma unroll
          for (int j = i; j < 3; ++j)
            Rg[sidx(i, j)] = 0.5 * (__dmul_rn(row3(gt, kk, i), d.d1[j]) + __dmul_rn(row3(gt, kk, j), d.d1[i]));
        const double trR = trace6(gi, Rg);
        const double ca = chi * alpha;
        if (TF_ONCE) {
#pragma unroll
          for (int r = 0; r < 6; ++r) SL(A_AT + r) += ca * Rg[r];
          ttr += ca * trR;
        } else {
#pragma unroll
          for (int r = 0; r < 6; ++r) SL(A_AT + r) += ca * (Rg[r] - gt[r] * trR * (1.0 / 3.0));
        }
      } else if (f == 2) {
        // ---------------- K: advection, KO, eq (8) -4/3 alpha gt^ij d_j K
        rK += __dadd_rn(advect<UPW>(s, c0, beta, d.d1, ih), d.ko);
        double gi[6];
        VALS_LD(TV_GI, gi);
#pragma unroll
        for (int i = 0; i < 3; ++i)
          SL(A_GT + i) += -(4.0 / 3.0) * alpha *
                          (gi[sidx(i, 0)] * d.d1[0] + gi[sidx(i, 1)] * d.d1[1] +
                           gi[sidx(i, 2)] * d.d1[2]);
      } else if (f >= 18) {
        const int q = f - 18;
        SL(A_AT + q) += __dadd_rn(advect<UPW>(s, c0, beta, d.d1, ih), d.ko);
      } else {  // 9..11: B
        const int kk = f - 9;
        SL(A_B + kk) = __dadd_rn(advect<UPW>(s, c0, beta, d.d1, ih), d.ko);
      }
    };
    // the per-point work of one staged field f (patch in s); a pair stage runs
    // it for both fields, in order
    auto point_work = [&](const double* __restrict__ s, const int f) __attribute__((always_inline)) {
    const int c0 = active ? int(tab_c0[tid]) : C_CENTRE;
    {
      if (!PRE && f >= 12 && f <= 17) {
        // ---------------- conformal metric gt_q: d gt, gt^lm d_lm gt, adv, KO
        const int q = f - 12;
        const Derivs d = derivs2(s, Tx, Ty, c0, ih, ko_scale);
        double gi[6];
        VALS_LD(TV_GI, gi);
#pragma unroll
        for (int k = 0; k < 3; ++k) SL(S0 + k * 6 + q) = d.d1[k];
        SL(A_AT + q) = trace6(gi, d.dd);   // (A_AT slot reused until the Christoffel block)
        SL(A_GAM + q) += __dadd_rn(advect<UPW>(s, c0, beta, d.d1, ih), d.ko);
        if (q == 5) christoffel(gi);
      } else if (f == 1) {
        // ---------------- chi: advection, KO, R^chi (eq 18-19), eq (8) chi term
        const Derivs d = derivs2(s, Tx, Ty, c0, ih, ko_scale);
        double gi[6], At[6], gt[6];
        VALS_LD(TV_GI, gi);
        VALS_LD(TV_AT, At);
        VALS_LD(TV_GT, gt);
#pragma unroll
        for (int k = 0; k < 3; ++k) dchi[k] = d.d1[k];
        rC += __dadd_rn(advect<UPW>(s, c0, beta, d.d1, ih), d.ko);
        double Rc[6];
#pragma unroll
        for (int i = 0; i < 3; ++i)
#pragma unroll
          for (int j = i; j < 3; ++j) {
            const int q = sidx(i, j);
            const double gd = SL(S0 + 0 * 6 + q) * dchi[0] + SL(S0 + 1 * 6 + q) * dchi[1] +
                              SL(S0 + 2 * 6 + q) * dchi[2];
            Rc[q] = (d.dd[q] - gd) * (0.5 * ichi) - dchi[i] * dchi[j] * (0.25 * ichi * ichi);
          }
        const double trR = trace6(gi, Rc);
        const double ca = chi * alpha;
        if (TF_ONCE) {
#pragma unroll
          for (int r = 0; r < 6; ++r) SL(A_AT + r) += ca * Rc[r];
          ttr += ca * trR;
        } else {
#pragma unroll
          for (int r = 0; r < 6; ++r) SL(A_AT + r) += ca * (Rc[r] - gt[r] * trR * (1.0 / 3.0));
        }
        // Gt^i += -3 alpha / chi At^ij d_j chi
        {
          double v[3];
          at_up_w(gi, At, dchi, v);
#pragma unroll
          for (int i = 0; i < 3; ++i) SL(A_GT + i) += -3.0 * alpha * ichi * v[i];
        }
      } else if (f == 0) {
        // ---------------- alpha: advection, KO, D_i D_j alpha (eqs 13-15)
        const Derivs d = derivs2(s, Tx, Ty, c0, ih, ko_scale);
        double gi[6], At[6], gt[6];
        VALS_LD(TV_GI, gi);
        VALS_LD(TV_AT, At);
        VALS_LD(TV_GT, gt);
        const double* da = d.d1;
        rA += __dadd_rn(advect<UPW>(s, c0, beta, da, ih), d.ko);
        // gt^kl d_l chi d_k alpha
        double gdd = 0.0;
#pragma unroll
        for (int k = 0; k < 3; ++k)
#pragma unroll
          for (int l = 0; l < 3; ++l) gdd += gi[sidx(k, l)] * dchi[l] * da[k];
        double DD[6];
#pragma unroll
        for (int i = 0; i < 3; ++i)
#pragma unroll
          for (int j = i; j < 3; ++j) {
            const int q = sidx(i, j);
            const double gk = SL(S0 + 0 * 6 + q) * da[0] + SL(S0 + 1 * 6 + q) * da[1] +
                              SL(S0 + 2 * 6 + q) * da[2];
            const double phys = gk - (0.5 * ichi) * (dchi[i] * da[j] + dchi[j] * da[i] - gt[q] * gdd);
            DD[q] = d.dd[q] - phys;
          }
        const double trD = trace6(gi, DD);
        rK += -chi * trD;
        if (TF_ONCE) {
#pragma unroll
          for (int r = 0; r < 6; ++r) SL(A_AT + r) += -chi * DD[r];
          ttr += -chi * trD;
        } else {
#pragma unroll
          for (int r = 0; r < 6; ++r) SL(A_AT + r) += -chi * (DD[r] - gt[r] * trD * (1.0 / 3.0));
        }
        {
          double v[3];
          at_up_w(gi, At, da, v);
#pragma unroll
          for (int i = 0; i < 3; ++i) SL(A_GT + i) += -2.0 * v[i];
        }
      } else if (f >= 6 && f <= 8) {
        // ---------------- beta^kk: Lie derivative terms, eq (2), eq (8) shift terms
        const int kk = f - 6;
        const Derivs d = derivs2(s, Tx, Ty, c0, ih, ko_scale);
        const double* db = d.d1;   // d_j beta^kk
        const double dbk = sel3(kk, db[0], db[1], db[2]);   // d_kk beta^kk
        SL(A_BETA + kk) += __dadd_rn(advect<UPW>(s, c0, beta, db, ih), d.ko);
        double gi[6], cal[3];
        VALS_LD(TV_GI, gi);
#pragma unroll
        for (int k = 0; k < 3; ++k) cal[k] = SL(A_B + k);
        // Lie derivative terms of gt and At (eq 10, w = -2/3) need all of d_j beta^k:
        // the first two beta stages park d_j beta^k in scratch slots S0+3.., the
        // last one applies  T_ik d_j b^k + T_kj d_i b^k - 2/3 T_ij d_k b^k  once
        if (kk < 2) {
#pragma unroll
          for (int j = 0; j < 3; ++j) SL(S0 + 3 + 3 * kk + j) = db[j];
        } else {
          double DB[3][3];   // DB[k][j] = d_j beta^k
#pragma unroll
          for (int k = 0; k < 2; ++k)
#pragma unroll
            for (int j = 0; j < 3; ++j) DB[k][j] = SL(S0 + 3 + 3 * k + j);
#pragma unroll
          for (int j = 0; j < 3; ++j) DB[2][j] = db[j];
          const double div = DB[0][0] + DB[1][1] + DB[2][2];
#pragma unroll
          for (int t = 0; t < 2; ++t) {
            const int ab = t == 0 ? A_GAM : A_AT;
            double T[6];
            VALS_LD(t == 0 ? TV_GT : TV_AT, T);
#pragma unroll
            for (int i = 0; i < 3; ++i)
#pragma unroll
              for (int j = i; j < 3; ++j) {
                const int q = sidx(i, j);
                double l = -(2.0 / 3.0) * T[q] * div;
#pragma unroll
                for (int k = 0; k < 3; ++k)
                  l += T[sidx(i, k)] * DB[k][j] + T[sidx(k, j)] * DB[k][i];
                SL(ab + q) += l;
              }
          }
        }
        rC = __fma_rn(-(2.0 / 3.0) * chi, dbk, rC);
        // Gt^kk += gt^jl d_jl beta^kk - CalGt^j d_j beta^kk
        SL(A_GT + kk) += trace6(gi, d.dd) - (cal[0] * db[0] + cal[1] * db[1] + cal[2] * db[2]);
        // Gt^i += 1/3 gt^ij d_j d_kk beta^kk + 2/3 CalGt^i d_kk beta^kk
#pragma unroll
        for (int i = 0; i < 3; ++i)
          SL(A_GT + i) += __fma_rn(1.0 / 3.0,
                                   __fma_rn(gi[sidx(i, 2)], row3(d.dd, kk, 2),
                                            __fma_rn(gi[sidx(i, 1)], row3(d.dd, kk, 1),
                                                     __dmul_rn(gi[sidx(i, 0)], row3(d.dd, kk, 0)))),
                                   __dmul_rn((2.0 / 3.0) * cal[i], dbk));
      } else {
        light_apply(s, f, derivs<false>(s, c0, ih, ko_scale));
      }
    }
    };
    if (SOMM && bwarp) {
      // radiative condition (reading R29) for the stage's field(s), parked in
      // TMEM; the epilogue uses it at points on a domain face (every thread
      // of a warp that has one stores: tcgen05.st is warp-wide)
      const int c0 = active ? int(tab_c0[tid]) : C_CENTRE;
      somm_park(m, oi, int(tab_p[tid]), s, c0, ih, f, tma + 2 * (6 * TV_SOMM + f));
      if (FUSED && stB(st) >= 0)
        somm_park(m, oi, int(tab_p[tid]), Tx + buf * STAGE_DBL, c0, ih, stB(st),
                  tma + 2 * (6 * TV_SOMM + stB(st)));
    }
    if (FUSED && !SOMM && stB(st) >= 0) {
      // a pair of light fields: both fields' derivatives first (one straight
      // line of 2 x 19 independent shared-memory loads, so the two fields'
      // latency chains overlap), then each field's algebra in the pair order
      // — the same arithmetic as two single stages
      const int c0 = active ? int(tab_c0[tid]) : C_CENTRE;
      {
        const double* sB = Tx + buf * STAGE_DBL;
        const Derivs dA = derivs<false>(s, c0, ih, ko_scale);
        const Derivs dB = derivs<false>(sB, c0, ih, ko_scale);
        light_apply(s, f, dA);
        light_apply(sB, stB(st), dB);
      }
    } else {
      point_work(s, f);
      if (FUSED && stB(st) >= 0) point_work(Tx + buf * STAGE_DBL, stB(st));
    }
    __syncthreads();  // everyone is done with this stage buffer
    if (FUSED) {
      if (st + 2 < NST) {
        gather_stage(buf, st + 2, st + 3 == NST ? en : -1);
      } else {
        if (st + 2 == NST && en >= 0) load_gidx(en);   // the current octant's gathers are issued
        if (en >= 0) gather_stage(buf, st + 2 - NST);
        else cp_async_commit();                         // (empty group keeps the count uniform)
      }
      continue;
    }
    // L2 prefetch one octant ahead: the next octant's field of this stage
    // (measured faster than prefetching the current octant at its start,
    // although some prefetched lines are evicted and re-read)
    if (tid == 32 && en >= 0)
      prefetch_l2(patches + int64_t(en) * PATCH_PITCH + ORD[st] * fstride);
    if (tid == 0) {
      if (st + 2 < NS)
        bulk_load(stage + buf * STAGE_DBL, pbase + ORD[st + 2] * fstride, STAGE_DBL * 8,
                  &bars[buf]);
      else if (en >= 0)   // the stream continues with the next octant's first fields
        bulk_load(stage + buf * STAGE_DBL,
                  patches + int64_t(en) * PATCH_PITCH + ORD[st + 2 - NS] * fstride,
                  STAGE_DBL * 8, &bars[buf]);
    }
  }

#ifdef DGR_RHS_TIMING
  if (tid == 0) {
    const long long t = clock64();
    atomicAdd(reinterpret_cast<unsigned long long*>(&g_stage_cycles[NF]),
              (unsigned long long)(t - t_last));
    t_last = t;
  }
#endif
  // ---- epilogue: undifferentiated terms, combine, store ----------------------
  const int p = tab_p[tid];
  {
    double gi[6], At[6], gtv[6], B[3];
    VALS_LD(TV_GI, gi);
    VALS_LD(TV_AT, At);
    if (TF_ONCE) VALS_LD(TV_GT, gtv);
    double ex[6];
    VALS_LD(TV_EX, ex);
    // (zip by the store: the DOF this point is the zip owner of, or -1)
    const int dz = __double2loint(ex[3]);
#pragma unroll
    for (int i = 0; i < 3; ++i)
      B[i] = ex[i];
    // At^k_j and At_ik At^k_j, At_ij At^ij
    double Am[3][3];
#pragma unroll
    for (int k = 0; k < 3; ++k)
#pragma unroll
      for (int j = 0; j < 3; ++j)
        Am[k][j] = gi[sidx(k, 0)] * At[sidx(0, j)] + gi[sidx(k, 1)] * At[sidx(1, j)] +
                   gi[sidx(k, 2)] * At[sidx(2, j)];
    double AA = 0.0;
#pragma unroll
    for (int i = 0; i < 3; ++i)
#pragma unroll
      for (int j = 0; j < 3; ++j) AA += Am[i][j] * Am[j][i];
    double r[NF];
    r[0] = rA - 2.0 * alpha * Kv;                                                 // (1)
    r[1] = rC + (2.0 / 3.0) * chi * alpha * Kv;                                   // (5)
    r[2] = rK + alpha * (AA + Kv * Kv * (1.0 / 3.0));                             // (7)
    const double fa = prm.lambda_f0 + prm.lambda_f1 * alpha;
#pragma unroll
    for (int i = 0; i < 3; ++i) {
      const double gbar = SL(A_GT + i);
      r[3 + i] = gbar + SL(S0 + i);                                               // (8)
      r[6 + i] = SL(A_BETA + i) + 0.75 * fa * B[i];                               // (2)
      r[9 + i] = gbar - prm.eta * B[i] + SL(A_B + i);                             // (3)
    }
#pragma unroll
    for (int i = 0; i < 3; ++i)
#pragma unroll
      for (int j = i; j < 3; ++j) {
        const int q = sidx(i, j);
        r[12 + q] = SL(A_GAM + q) - 2.0 * alpha * At[q];                          // (4)
        const double AAij = At[sidx(i, 0)] * Am[0][j] + At[sidx(i, 1)] * Am[1][j] +
                            At[sidx(i, 2)] * Am[2][j];
        const double atf = TF_ONCE ? SL(A_AT + q) - gtv[q] * ttr * (1.0 / 3.0) : SL(A_AT + q);
        r[18 + q] = atf + alpha * (Kv * At[q] - 2.0 * AAij);                        // (6)
      }
    if (SOMM && bwarp) {
      // points on a domain face: the radiative condition replaces the whole
      // right-hand side (reading R29)
      tm_st_wait();
      double rv[NF];
#pragma unroll
      for (int b = 0; b < 4; ++b) VALS_LD(TV_SOMM + b, rv + 6 * b);
      if (bpt) {
#pragma unroll
        for (int f = 0; f < NF; ++f) r[f] = rv[f];
      }
    }
    double* out = rhs_oct + int64_t(e) * NPT + p;
    const int64_t ostr = no * NPT;
    if (rhs_dof && prm.rk_stage >= 0) {
      // the RK4 stage update of the owned DOF dz, in batches of RKB fields (an
      // L2 prefetch of the u_n / acc rows two stages ahead measured slower:
      // 26.30 vs 26.69 ms per C3 step, its 48 prefetches per thread cost more)
      if (dz >= 0) {
        const int S = prm.rk_stage;
        const double dt = prm.rk_dt;
        const int64_t ds64 = m.dof_stride;
#pragma unroll
        for (int f0 = 0; f0 < NF; f0 += RKB) {
          double un[RKB], ac[RKB];
#pragma unroll
          for (int j = 0; j < RKB; ++j) {
            const int64_t i = (f0 + j) * ds64 + dz;
            un[j] = S <= 2 ? __ldcs(prm.rk_un + i) : 0.0;
            ac[j] = S >= 1 ? __ldcs(prm.rk_acc + i) : 0.0;
          }
#pragma unroll
          for (int j = 0; j < RKB; ++j) {
            const int64_t i = (f0 + j) * ds64 + dz;
            const double k = r[f0 + j];
            if (S == 0) {
              prm.rk_acc[i] = __fma_rn(dt / 6.0, k, un[j]);
              prm.rk_us[i] = __fma_rn(dt / 2.0, k, un[j]);
            } else if (S == 1) {
              prm.rk_acc[i] = __fma_rn(dt / 3.0, k, ac[j]);
              prm.rk_us[i] = __fma_rn(dt / 2.0, k, un[j]);
            } else if (S == 2) {
              prm.rk_acc[i] = __fma_rn(dt / 3.0, k, ac[j]);
              prm.rk_us[i] = __fma_rn(dt, k, un[j]);
            } else {
              prm.rk_out[i] = __fma_rn(dt / 6.0, k, ac[j]);
            }
          }
        }
      }
    } else if (rhs_dof) {
      if (dz >= 0) {
#pragma unroll
        for (int f = 0; f < NF; ++f) st_out(&rhs_dof[f * int64_t(m.dof_stride) + dz], r[f]);
      }
    } else if (active) {
#pragma unroll
      for (int f = 0; f < NF; ++f) out[f * ostr] = r[f];
    }
  }
  }  // octant loop
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (tid < 32)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(*tm_base),
                 "n"(SOMM ? TM_COLS_SOMM : TM_COLS)
                 : "memory");
#undef SL
#undef VALS_LD
#undef VALS_ST
}

// ---------------------------------------------------------------------------
// Metric pre-pass (DESIGN.md §8c item 1): the six conformal-metric fields
// gt_q (second derivatives) without any cross-field state, so two CTAs fit on
// an SM twice (22 warps instead of 11; three CTAs per SM, at 56 registers,
// measured slower: 1.99 vs 1.53 ms on C3).  Per interior point it writes 30 values to
// pre[c][n_owned][352] (indexed by the thread of the point, as in k_rhs):
//   c = 6k + q   d_k gt_q                       (k = 0..2, q = 0..5)
//   c = 18 + q   gt^lm d_l d_m gt_q             (the -1/2 term of Rt, eq 17)
//   c = 24 + q   beta^k d_k gt_q + KO(gt_q)     (eq 4 advection + dissipation)
// which k_rhs<..., PRE = true> reads instead of staging the gt fields itself.
// Same stencils, same gather/extrapolation and same arithmetic order as the
// gt stages of k_rhs, so both paths give bit-identical results.
constexpr int NPRE = 30;   // rows per point (api.cu allocates pre_rows() of them)
int pre_rows() { return NPRE; }
#ifndef DGR_PRE_NBUF
#define DGR_PRE_NBUF 2   // (A/B r3ag: 27.01 -> 26.91 ms per C3 step with 2)
#endif
// stage ring depth of the pre-pass: 3 = one barrier per field (the gather of
// field g+2 goes into the buffer of g-1 after the start barrier); 2 = a second
// barrier per field, 17.6 KB less shared memory per CTA (more L1)
constexpr int PRE_NBUF = DGR_PRE_NBUF;
constexpr size_t PRE_SMEM_BYTES = size_t(PRE_NBUF) * STAGE_DBL * 8 + size_t(TX_N + TY_N) * 8 +
                                  16 + size_t(RT) * 4 + size_t(3) * RT * 2;

// Fused path only (patches gathered from u and the slots).  Three-deep stage
// ring: the CTA barrier that releases stage g's data also proves every thread
// is done with stage g-1, whose buffer then receives stage g+2 (two stages of
// latency cover, two barriers per field).
template <bool UPW>
__global__ void __launch_bounds__(RT, 2)
    k_gt_pre(DevMesh m, const double* __restrict__ patches, double* __restrict__ pre,
             RhsParams prm, int first, int count) {
  extern __shared__ __align__(128) double smem[];
  double* stage = smem;                           // [PRE_NBUF][STAGE_DBL]
  double* Tx = stage + PRE_NBUF * STAGE_DBL;      // [TX_N]
  double* Ty = Tx + TX_N;                         // [TY_N]
  // the octant-to-come's anchor and each thread's o2s index (cp.async, as k_rhs)
  int4* sm_oi = reinterpret_cast<int4*>(Ty + TY_N);
  int32_t* tab_cv = reinterpret_cast<int32_t*>(sm_oi + 1);
  int16_t* tab_c0 = reinterpret_cast<int16_t*>(tab_cv + RT);
  int16_t* tab_p = tab_c0 + RT;
  int16_t* tab_d1b = tab_p + RT;
  const int tid = threadIdx.x;
  {
    const int pp = g_perm[tid];
    const int q = pp >= 0 ? pp : 0;
    tab_c0[tid] = pp >= 0 ? int16_t((q % 7 + 3) + 13 * ((q / 7) % 7 + 3) + 169 * (q / 49 + 3)) : -1;
    tab_p[tid] = int16_t(q);
    tab_d1b[tid] = g_d1b[tid];
  }
  const int64_t no = m.n_owned;
  const int64_t fstride = m.dof_stride;
  const int32_t ds = int32_t(m.dof_stride);
  const int32_t* ol = m.olist + first;
  int li = blockIdx.x;
  if (li >= count) return;
  int e = ol[li];
  int gidx[GJ];
  int gdst[GJ];
  auto load_gidx = [&](int oct) {
    const int32_t* gm = m.gmap_s + int64_t(oct) * GM_PITCH;
    const int16_t* gd = m.gdst + int64_t(oct) * GM_PITCH;
#pragma unroll
    for (int j = 0; j < GJ; ++j) {
      const int pt = tid + RT * j;
      gidx[j] = pt < NPATCH ? max(__ldg(gm + pt), 0) : -1;
      gdst[j] = pt < NPATCH ? int(__ldg(gd + pt)) : 0;
    }
  };
  auto gather = [&](double* dst, int f, int oct_next = -1) {
    // (gt fields: the three slabs the stencils and the D1 pass read)
    const uint32_t d0 = smem_u32(dst);
    const double* uf = patches + f * fstride;
    const double* af = m.aux + f * m.aux_stride - m.dof_stride;
#pragma unroll
    for (int j = 0; j < GJ; ++j)
      if (tid + RT * j < G_SLABS) cp_async8(d0 + 8 * gdst[j], uf, af, gidx[j], ds);
    if (oct_next >= 0) {   // (lands before that octant's prologue)
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(tab_cv + tid)),
                   "l"(m.o2s + int64_t(oct_next) * NPT + int(tab_p[tid]))
                   : "memory");
      if (tid == 0)
        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(smem_u32(sm_oi)),
                     "l"(m.oct + oct_next)
                     : "memory");
    }
    cp_async_commit();
  };
  tab_cv[tid] = __ldg(m.o2s + int64_t(e) * NPT + int(tab_p[tid]));
  if (tid == 0) *sm_oi = m.oct[e];
  __syncthreads();
  load_gidx(e);
  gather(stage, 12);
  gather(stage + STAGE_DBL, 13);
  uint32_t g = 0;
  for (; li < count; li += gridDim.x) {
    e = ol[li];
    const int en = li + int(gridDim.x) < count ? ol[li + gridDim.x] : -1;
    const int c0 = tab_c0[tid];
    const int p = tab_p[tid];
    const int4 oi = *sm_oi;
    int omask = 0;
    if (!m.periodic) {
      const int nside = 1 << m.D, sd = 1 << (m.D - oi.w);
      omask = (oi.x == 0) | ((oi.y == 0) << 1) | ((oi.z == 0) << 2) | ((oi.x + sd == nside) << 3) |
              ((oi.y + sd == nside) << 4) | ((oi.z + sd == nside) << 5);
    }
    if (en >= 0 && tid == 32) {   // next octant's gather rows (gmap_s, gdst) into L2
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(m.gmap_s + int64_t(en) * GM_PITCH),
                   "r"(uint32_t(GM_PITCH * 4))
                   : "memory");
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(m.gdst + int64_t(en) * GM_PITCH),
                   "r"(uint32_t(GM_PITCH * 2))
                   : "memory");
    }
    const double ih = (6.0 * double(int64_t(1) << oi.w)) / m.width;   // 1/h
    const double ko_scale = prm.ko_sigma * ih * (1.0 / 64.0);
    // values at the point: gt (for gt^ij) and beta (advection)
    double gi[6] = {0, 0, 0, 0, 0, 0}, beta[3] = {0, 0, 0};
    if (c0 >= 0) {
      const int cv = tab_cv[tid];
      auto own = [&](int f) -> double {
        return cv < ds ? __ldg(patches + f * fstride + cv) : __ldg(m.aux + f * m.aux_stride + (cv - ds));
      };
      double gq[6];
#pragma unroll
      for (int q = 0; q < 6; ++q) gq[q] = own(12 + q);
#pragma unroll
      for (int i = 0; i < 3; ++i) beta[i] = own(6 + i);
      const double a00 = gq[3] * gq[5] - gq[4] * gq[4];
      const double a01 = gq[2] * gq[4] - gq[1] * gq[5];
      const double a02 = gq[1] * gq[4] - gq[2] * gq[3];
      const double det = gq[0] * a00 + gq[1] * a01 + gq[2] * a02;
      const double idet = 1.0 / det;
      gi[0] = a00 * idet;
      gi[1] = a01 * idet;
      gi[2] = a02 * idet;
      gi[3] = (gq[0] * gq[5] - gq[2] * gq[2]) * idet;
      gi[4] = (gq[1] * gq[2] - gq[0] * gq[4]) * idet;
      gi[5] = (gq[0] * gq[3] - gq[1] * gq[1]) * idet;
    }
    // rows indexed by thread (the same thread -> point map as k_rhs): coalesced
    double* out = pre + int64_t(e) * RT + tid;
    const int64_t ostr = no * RT;
    for (int q = 0; q < 6; ++q, ++g) {
      const int buf = g % PRE_NBUF;
      cp_async_wait1();   // this thread's copies of stage g (g+1 may be in flight)
      __syncthreads();    // everyone's; and everyone is done with stage g-1
      auto issue_next = [&]() {
        // stage g+2 into the buffer of stage g-1 (ring of 3) / of stage g (ring of 2)
        double* dst = stage + ((g + 2) % PRE_NBUF) * STAGE_DBL;
        if (q + 2 < 6) {
          gather(dst, 12 + q + 2, q == 3 ? en : -1);
        } else {
          if (q == 4 && en >= 0) load_gidx(en);
          if (en >= 0) gather(dst, 12 + q + 2 - 6);
          else cp_async_commit();
        }
      };
      if (PRE_NBUF == 3) issue_next();
      double* sw = stage + buf * STAGE_DBL;
      if (omask) {
        for (int a = 0; a < 3; ++a) {
          const int sa = a == 0 ? 1 : (a == 1 ? 13 : 169);
          const int sb = a == 0 ? 13 : 1, sc = a == 2 ? 13 : 169;
          const int b_ax = a == 0 ? 1 : 0, c_ax = a == 2 ? 1 : 2;
          for (int side = 0; side < 2; ++side) {
            if (!((omask >> (a + 3 * side)) & 1)) continue;
            for (int idx = tid; idx < 3 * 169; idx += RT) {
              const int k3 = idx % 3, uv = idx / 3;
              const int cb = uv % 13, cc = uv / 13;
              if (b_ax > a && ((cb < 3 && ((omask >> b_ax) & 1)) || (cb > 9 && ((omask >> (3 + b_ax)) & 1))))
                continue;
              if (c_ax > a && ((cc < 3 && ((omask >> c_ax) & 1)) || (cc > 9 && ((omask >> (3 + c_ax)) & 1))))
                continue;
              const int ia = side == 0 ? k3 : 10 + k3;
              const int base = cb * sb + cc * sc;
              double acc = 0.0;
              if (side == 0) {
                const double* w = c_rWEXT + (2 - ia) * 7;
#pragma unroll
                for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], sw[base + (3 + mm) * sa], acc);
              } else {
                const double* w = c_rWEXT + (ia - 10) * 7;
#pragma unroll
                for (int mm = 0; mm < 7; ++mm) acc = fma(w[mm], sw[base + (9 - mm) * sa], acc);
              }
              sw[base + ia * sa] = acc;
            }
          }
          __syncthreads();
        }
      }
      const double* s = sw;
      // cooperative D1 pass (as in k_rhs)
      d1_pass(s, Tx, Ty, tid, tab_d1b);
      __syncthreads();
      if (c0 >= 0) {
        const Derivs d = derivs2(s, Tx, Ty, c0, ih, ko_scale);
#pragma unroll
        for (int k = 0; k < 3; ++k) st_out(&out[(6 * k + q) * ostr], d.d1[k]);
        st_out(&out[(18 + q) * ostr], trace6(gi, d.dd));
        st_out(&out[(24 + q) * ostr], __dadd_rn(advect<UPW>(s, c0, beta, d.d1, ih), d.ko));
      }
      if (PRE_NBUF == 2) {
        __syncthreads();   // everyone is done with this stage buffer
        issue_next();
      }
    }
  }
}

size_t rhs_smem_bytes() { return SMEM_BYTES; }

#ifdef DGR_RHS_TIMING
}  // namespace dgr
// experiment builds only (tools/rhs_stage_profile.py): summed cycles of CTA
// thread 0 per stage slot; out[NF + 1], reset after reading
extern "C" int dgr_debug_rhs_stage_cycles(long long* out) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out, dgr::g_stage_cycles, sizeof(long long) * (dgr::NF + 1));
  long long zero[dgr::NF + 2] = {0};
  cudaMemcpyToSymbol(dgr::g_stage_cycles, zero, sizeof(zero));
  return 0;
}
namespace dgr {
#endif

void upload_rhs_tables(const double* wext) {
  cudaMemcpyToSymbol(c_rWEXT, wext, sizeof(double) * 21);
  int16_t perm[RT];
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
  cudaMemcpyToSymbol(g_perm, perm, sizeof(perm));
  // D1-pass lines: per kind, fill each half-warp with lines of distinct b mod 16
  // (greedy, the most frequent residues first)
  int16_t d1b[RT];
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
  cudaMemcpyToSymbol(g_d1b, d1b, sizeof(d1b));
}

template <bool U>
static void launch_rhs_t(const DevMesh& m, const double* patches, double* rhs_oct,
                         const RhsParams& p, bool fused, bool somm, int a, int c, int grid,
                         int64_t cap, cudaStream_t s, double* pre, double* rhs_dof) {
  if (fused && pre) {
    // metric pre-pass (two CTAs per SM), then the 18 remaining fields
    const int64_t cap2 = 2 * cap;
    const int grid2 = int(c < cap2 ? c : cap2);
    k_gt_pre<U><<<grid2, RT, PRE_SMEM_BYTES, s>>>(m, patches, pre, p, a, c);
    if (somm)
      k_rhs<true, true, true, U><<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, pre, rhs_dof);
    else
      k_rhs<true, false, true, U><<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, pre, rhs_dof);
  } else if (fused && !somm)
    k_rhs<true, false, false, U><<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, nullptr, rhs_dof);
  else if (fused)
    k_rhs<true, true, false, U><<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, nullptr, rhs_dof);
  else if (!somm)
    k_rhs<false, false, false, U><<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, nullptr, nullptr);
  else
    k_rhs<false, true, false, U><<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, nullptr, nullptr);
}

void launch_rhs(const DevMesh& m, const double* patches, double* rhs_oct, const RhsParams& p,
                bool fused, int64_t first, int64_t count, int leave_sm, cudaStream_t s,
                double* pre, double* rhs_dof) {
  if (count <= 0) return;
  static std::atomic<bool> done[MAX_DEVICES];
  if (first_on_device(done)) {
    const int sb = int(SMEM_BYTES);
#define DGR_ATTR(F, S, P, U) \
    cudaFuncSetAttribute(k_rhs<F, S, P, U>, cudaFuncAttributeMaxDynamicSharedMemorySize, sb);
    DGR_ATTR(false, false, false, false) DGR_ATTR(true, false, false, false)
    DGR_ATTR(false, true, false, false) DGR_ATTR(true, true, false, false)
    DGR_ATTR(true, false, true, false) DGR_ATTR(false, false, false, true)
    DGR_ATTR(true, false, false, true) DGR_ATTR(false, true, false, true)
    DGR_ATTR(true, true, false, true) DGR_ATTR(true, false, true, true)
    DGR_ATTR(true, true, true, false) DGR_ATTR(true, true, true, true)
#undef DGR_ATTR
    cudaFuncSetAttribute(k_gt_pre<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(PRE_SMEM_BYTES));
    cudaFuncSetAttribute(k_gt_pre<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(PRE_SMEM_BYTES));
  }
  const int n_sm = sm_count();
  // persistent: one CTA per SM (227 KB of shared memory each)
  const int64_t cap = leave_sm > 0 && n_sm - leave_sm > 0 ? n_sm - leave_sm : n_sm;
  const int grid = int(count < cap ? count : cap);
  const bool somm = p.sommerfeld && !m.periodic;
  const int a = int(first), c = int(count);
  if (p.upwind)
    launch_rhs_t<true>(m, patches, rhs_oct, p, fused, somm, a, c, grid, cap, s, pre, rhs_dof);
  else
    launch_rhs_t<false>(m, patches, rhs_oct, p, fused, somm, a, c, grid, cap, s, pre, rhs_dof);
}

}  // namespace dgr
