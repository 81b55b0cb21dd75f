// k_rhs_fi: every instantiation of the RHS kernel except the default one
// (rhs_kernel.cu), with point_work force-inlined.  A separate translation unit
// so the forced inlining cannot change the default kernel's code (see
// rhs_kernel.cu); the kernel template is rhs_kernel_body.cuh.
#include "rhs_common.cuh"

namespace dgr {

#define DGR_KRHS k_rhs_fi
#define DGR_PW_INLINE __attribute__((always_inline))
#include "rhs_kernel_body.cuh"
#undef DGR_KRHS
#undef DGR_PW_INLINE

void upload_rhs_tables_fi(const double* wext) { upload_tables_here(wext); }

template <bool U>
static void launch_fi_t(const DevMesh& m, const double* patches, double* rhs_oct,
                        const RhsParams& p, bool fused, bool somm, bool pre_on, int a, int c,
                        int grid, cudaStream_t s, const double* pre, double* rhs_dof) {
  const int sb = int(SMEM_BYTES);
  auto go = [&](auto kern, const double* pr, double* rd) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, sb);
    kern<<<grid, RT, SMEM_BYTES, s>>>(m, patches, rhs_oct, p, a, c, pr, rd);
  };
  if (pre_on && somm)
    go(k_rhs_fi<true, true, true, U>, pre, rhs_dof);
  else if (pre_on)
    go(k_rhs_fi<true, false, true, U>, pre, rhs_dof);
  else if (fused && !somm)
    go(k_rhs_fi<true, false, false, U>, nullptr, rhs_dof);
  else if (fused)
    go(k_rhs_fi<true, true, false, U>, nullptr, rhs_dof);
  else if (!somm)
    go(k_rhs_fi<false, false, false, U>, nullptr, nullptr);
  else
    go(k_rhs_fi<false, true, false, U>, nullptr, nullptr);
}

void launch_rhs_fi(const DevMesh& m, const double* patches, double* rhs_oct, const RhsParams& p,
                   bool fused, bool somm, bool pre_on, bool upw, int a, int c, int grid,
                   cudaStream_t s, const double* pre, double* rhs_dof) {
  if (upw)
    launch_fi_t<true>(m, patches, rhs_oct, p, fused, somm, pre_on, a, c, grid, s, pre, rhs_dof);
  else
    launch_fi_t<false>(m, patches, rhs_oct, p, fused, somm, pre_on, a, c, grid, s, pre, rhs_dof);
}

}  // namespace dgr
