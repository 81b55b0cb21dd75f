// The BSSN RHS kernel template (rhs_kernel.cu includes this file twice:
// DGR_KRHS names the kernel, DGR_PW_INLINE is point_work's inlining attribute;
// no include guard on purpose).  Everything it uses is defined in
// rhs_kernel.cu before the inclusion.
template <bool FUSED, bool SOMM, bool PRE, bool UPW>
__global__ void __launch_bounds__(RT, 1)
    DGR_KRHS(DevMesh m, const double* __restrict__ patches, double* __restrict__ rhs_oct,
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
    auto point_work = [&](const double* __restrict__ s, const int f) DGR_PW_INLINE {
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
