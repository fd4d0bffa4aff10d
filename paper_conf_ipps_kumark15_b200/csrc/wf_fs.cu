// wf_fs.cu -- wavefront_kernel instantiations for CellFS (generated layout, see wavefront_launch.cuh).
// Compiled with --fmad=false: the FS pull form must never be contracted to FFMA (R5).
#include "wavefront_launch.cuh"
namespace lddp {
int wf_dispatch_fs(int op, int variant, bool table, const FillParams* p, int grid, cudaStream_t s) {
  LDDP_WF_CASE(CellFS, WF_K_R1, 1, 2, 2, true)
  LDDP_WF_CASE(CellFS, WF_K_R2, 2, 2, 2, true)
  LDDP_WF_CASE(CellFS, WF_K_R1_E1, 1, 2, 1, true)
  (void)op; (void)p; (void)grid; (void)s;
  return -1;
}
}  // namespace lddp
