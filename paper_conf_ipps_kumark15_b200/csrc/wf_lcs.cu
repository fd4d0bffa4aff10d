// wf_lcs.cu -- wavefront_kernel instantiations for CellLCS (generated layout, see wavefront_launch.cuh).
#include "wavefront_launch.cuh"
namespace lddp {
int wf_dispatch_lcs(int op, int variant, bool table, const FillParams* p, int grid, cudaStream_t s) {
  LDDP_WF_CASE(CellLCS, WF_A_R4_S0, 4, 0, 2, false)
  LDDP_WF_CASE(CellLCS, WF_A_R2_S1, 2, 1, 1, false)
  LDDP_WF_CASE(CellLCS, WF_A_R2_S1, 2, 1, 1, true)
  LDDP_WF_CASE(CellLCS, WF_A_R8_S1, 8, 1, 1, false)
  LDDP_WF_CASE(CellLCS, WF_A_R4_S0, 4, 0, 2, true)
  LDDP_WF_CASE(CellLCS, WF_K_R1, 1, 2, 2, false)
  LDDP_WF_CASE(CellLCS, WF_K_R2, 2, 2, 2, false)
  LDDP_WF_CASE(CellLCS, WF_K_R1, 1, 2, 2, true)
  LDDP_WF_CASE(CellLCS, WF_K_R2, 2, 2, 2, true)
  (void)op; (void)p; (void)grid; (void)s;
  return -1;
}
}  // namespace lddp
