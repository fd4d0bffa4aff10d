// invl.cu -- launchers of the inverted-L kernel (invl.cuh; also instantiated by
// include/lddp_user.cuh) for DIAG_MAXPLUS and its mirror twin ANTIDIAG_MAXPLUS.
#include <cstdlib>

#include "invl.cuh"

namespace lddp {

template <class F, bool MIRROR>
static cudaError_t launch_il(const FillParams& p, int grid, cudaStream_t s) {
  // rows per register block (two blocks in flight per warp): LDDP_INVL_BLOCK = 8 / 16 / 24 / 32 (sweeps)
  static const int blk = [] { const char* e = getenv("LDDP_INVL_BLOCK"); return e ? atoi(e) : kInvlBlock; }();
  if (p.table != nullptr)
    invl_kernel<F, true, MIRROR><<<grid, kInvlWarps * 32, 0, s>>>(p);
  else if (blk == 32)
    invl_kernel<F, false, MIRROR, 32><<<grid, kInvlWarps * 32, 0, s>>>(p);
  else if (blk == 8)
    invl_kernel<F, false, MIRROR, 8><<<grid, kInvlWarps * 32, 0, s>>>(p);
  else if (blk == 24)
    invl_kernel<F, false, MIRROR, 24><<<grid, kInvlWarps * 32, 0, s>>>(p);
  else
    invl_kernel<F, false, MIRROR><<<grid, kInvlWarps * 32, 0, s>>>(p);
  return cudaGetLastError();
}

// func 4 DIAG_MAXPLUS (Inverted-L) and 8 ANTIDIAG_MAXPLUS (its mirror twin, the same cell on the
// mirrored grid, mirror = true)
cudaError_t launch_invl(int func, const FillParams& p, int grid, bool mirror, cudaStream_t s) {
  if (func != 4 && func != 8) return cudaErrorInvalidValue;
  return mirror ? launch_il<CellDiagMaxPlus, true>(p, grid, s) : launch_il<CellDiagMaxPlus, false>(p, grid, s);
}

}  // namespace lddp
