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
#include "rhs_common.cuh"

namespace dgr {

// FUSED = false: `patches` is the 13^3 patch buffer [24][n_owned][PATCH_PITCH]
// (bulk copies).  FUSED = true: `patches` is the state u and every patch is
// gathered straight from u and the interpolation slots through m.gmap with
// 8-byte cp.async (the unzip fused into the RHS), and
// points outside a non-periodic domain are extrapolated in shared memory with
// the same arithmetic as k_unzip.
// SOMM: radiative outer boundary (reading R29) compiled in (a separate
// instantiation, so the default path carries none of its registers).
// UPW: lopsided advective derivatives (reading R9u, dgr_params.upwind) compiled in
// k_rhs (this translation unit) is the default instantiation (fused, metric
// pre-pass, no radiative boundary, centred advection) and leaves point_work's
// inlining to nvcc; k_rhs_fi (rhs_kernel_fi.cu: every other instantiation, a
// separate translation unit so its forced inlining cannot change this one's
// code) forces it — outlined there, its captured state lived in local memory
// (C3: 65-72 instead of 27-31 ms per step) — while in the default
// instantiation forcing it costs 8 B of spills and 1.2%
#define DGR_KRHS k_rhs
#define DGR_PW_INLINE
#include "rhs_kernel_body.cuh"
#undef DGR_KRHS
#undef DGR_PW_INLINE

// (every instantiation of k_rhs is compiled in this unit, although only the
// default one is launched: with only that one, nvcc's code for it differs —
// 40 B instead of 32 B of spills, 1.3% slower on C3)
void* rhs_kernel_instances[] = {
    (void*)k_rhs<false, false, false, false>, (void*)k_rhs<true, false, false, false>,
    (void*)k_rhs<false, true, false, false>,  (void*)k_rhs<true, true, false, false>,
    (void*)k_rhs<true, false, true, false>,   (void*)k_rhs<false, false, false, true>,
    (void*)k_rhs<true, false, false, true>,   (void*)k_rhs<false, true, false, true>,
    (void*)k_rhs<true, true, false, true>,    (void*)k_rhs<true, false, true, true>,
    (void*)k_rhs<true, true, true, false>,    (void*)k_rhs<true, true, true, true>};

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

void upload_rhs_tables_fi(const double* wext);   // rhs_kernel_fi.cu
void upload_rhs_tables(const double* wext) {
  upload_tables_here(wext);
  upload_rhs_tables_fi(wext);
}

// rhs_kernel_fi.cu: k_rhs_fi<fused, somm, pre, upw> on (a, c) with `grid` CTAs
void launch_rhs_fi(const DevMesh& m, const double* patches, double* rhs_oct, const RhsParams& p,
                   bool fused, bool somm, bool pre_on, bool upw, int a, int c, int grid,
                   cudaStream_t s, const double* pre, double* rhs_dof);

void launch_rhs(const DevMesh& m, const double* patches, double* rhs_oct, const RhsParams& p,
                bool fused, int64_t first, int64_t count, int leave_sm, cudaStream_t s,
                double* pre, double* rhs_dof) {
  if (count <= 0) return;
  static std::atomic<bool> done[MAX_DEVICES];
  if (first_on_device(done)) {
    const int sb = int(SMEM_BYTES);
    cudaFuncSetAttribute(k_rhs<true, false, true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sb);
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
  const bool upw = p.upwind != 0;
  const int a = int(first), c = int(count);
  if (fused && pre) {
    // metric pre-pass (two CTAs per SM), then the 18 remaining fields
    const int64_t cap2 = 2 * cap;
    const int grid2 = int(c < cap2 ? c : cap2);
    if (upw)
      k_gt_pre<true><<<grid2, RT, PRE_SMEM_BYTES, s>>>(m, patches, pre, p, a, c);
    else
      k_gt_pre<false><<<grid2, RT, PRE_SMEM_BYTES, s>>>(m, patches, pre, p, a, c);
  }
  if (fused && pre && !somm && !upw)
    k_rhs<true, false, true, false><<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, pre, rhs_dof);
  else
    launch_rhs_fi(m, patches, rhs_oct, p, fused, somm, fused && pre, upw, a, c, grid, s, pre,
                  fused ? rhs_dof : nullptr);
}

}  // namespace dgr
