// wf_minpath3.cu -- wavefront_kernel instantiations for CellMinPath3 (generated layout, see wavefront_launch.cuh).
#include "wavefront_launch.cuh"
namespace lddp {
int wf_dispatch_minpath3(int op, int variant, bool table, const FillParams* p, int grid, cudaStream_t s) {
  LDDP_WF_CASE(CellMinPath3, WF_K_R1, 1, 2, 2, false)
  LDDP_WF_CASE(CellMinPath3, WF_K_R2, 2, 2, 2, false)
  LDDP_WF_CASE(CellMinPath3, WF_K_R1, 1, 2, 2, true)
  LDDP_WF_CASE(CellMinPath3, WF_K_R2, 2, 2, 2, true)
  (void)op; (void)p; (void)grid; (void)s;
  return -1;
}
}  // namespace lddp
