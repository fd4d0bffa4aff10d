// invl.cu -- launchers of the inverted-L kernel (invl.cuh; also instantiated by
// include/lddp_user.cuh) for DIAG_MAXPLUS and its mirror twin ANTIDIAG_MAXPLUS.
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include <cuda.h>
#include <cudaTypedefs.h>

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

// ---------------------------------------------------------------------------------------------
// TMA-staged variant (default for DIAG_MAXPLUS / ANTIDIAG_MAXPLUS without TABLE, grid pitch
// % 4 == 0): each warp streams its 32 diagonals as 2-D tensor boxes of 32 rows x 68 columns --
// the box that holds the parallelogram rows [i0, i0+32) x columns [i0+d0, i0+d0+63), its first
// column rounded down to a 16-byte multiple (the TMA unit faults otherwise) -- into a
// 3-slot shared ring (one lane issues cp.async.bulk.tensor, completion on an mbarrier per slot),
// two boxes in flight while the third is evaluated.  Lane l reads row u of a box at column
// u + l + sh (bank (5u + l + sh) mod 32: conflict-free).  Out-of-table box elements are zero-filled by the TMA
// unit.  Warp w evaluates diagonal groups w and w + NG/2 in turn: for a square table their chain
// lengths add up to the side, so every warp does the same work and all of them are resident.
// ---------------------------------------------------------------------------------------------
namespace {
constexpr int kItR = 32;      // rows per box
constexpr int kItX = 68;      // box columns: 63 + up to 3 of alignment (a box's x must be a 16-byte multiple)
constexpr int kItNB = 3;      // ring slots per warp
constexpr int kItWarps = 4;
constexpr size_t kItSmem = (size_t)kItWarps * kItNB * kItR * kItX * 4 + (size_t)kItWarps * kItNB * 8;

__device__ __forceinline__ void it_box(uint32_t dst, const CUtensorMap* tmap, int x, int y, uint32_t bar) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(kItR * kItX * 4)
               : "memory");
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(x), "r"(y), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void it_wait(uint32_t bar, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(bar), "r"(parity)
        : "memory");
  }
}
}  // namespace

template <bool MIRROR>
__global__ void __launch_bounds__(kItWarps * 32) invl_tma_kernel(const FillParams p, const __grid_constant__ CUtensorMap tmap_) {
  using F = CellDiagMaxPlus;
  using T = int32_t;
  extern __shared__ __align__(128) unsigned char it_smem[];
  const CUtensorMap* tmap = &tmap_;
  const int lane = threadIdx.x & 31;
  const int wl = threadIdx.x >> 5;
  const int64_t H = p.rows;
  const int W = p.cols;
  const int64_t dlo0 = p.diag_lo, dhi0 = p.diag_hi;
  const int64_t NG = (dhi0 - dlo0 + 31) / 32;
  const int64_t NP = (NG + 1) / 2;
  const uint32_t ring = smem_u32(it_smem) + (uint32_t)(wl * kItNB * kItR * kItX * 4);
  const uint32_t bar0 = smem_u32(it_smem + (size_t)kItWarps * kItNB * kItR * kItX * 4) + wl * kItNB * 8;
  if (lane == 0) {
    for (int k = 0; k < kItNB; ++k) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar0 + 8 * k) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  uint32_t nissue = 0, nuse = 0;   // boxes issued / consumed by this warp (slot = n % NB, parity = n / NB)
  const int64_t gw0 = (int64_t)blockIdx.x * kItWarps + wl;
  const int64_t gstride = (int64_t)gridDim.x * kItWarps;
  for (int64_t w = gw0; w < NP; w += gstride) {
#pragma unroll 1
    for (int h = 0; h < 2; ++h) {
      const int64_t g = w + h * NP;
      if (g >= NG) break;
      const int64_t d0 = dlo0 + g * 32;
      const int64_t d = d0 + lane;
      const bool live = d < dhi0;
      const int64_t dhi = min(dhi0 - 1, d0 + 31);
      const int64_t ibeg = max((int64_t)0, -dhi);
      const int64_t iend = min(H, (int64_t)W - d0);
      const int64_t ia = max((int64_t)0, -d), ib = min(H, (int64_t)W - d);
      T v = MIRROR ? T(0) : (d >= 0 ? F::top(p, (int)d - 1 + p.col0) : F::left(p, -d - 1));
      const int nbox = (int)((iend - ibeg + kItR - 1) / kItR);
      // the TMA box's first column must be 16-byte aligned: shift it left by sh (constant over the
      // group: consecutive boxes start 32 rows = 32 columns apart)
      const int64_t x0 = MIRROR ? (int64_t)W - 1 - (ibeg + d0 + 62) : ibeg + d0;
      const int sh = (int)(((x0 % 4) + 4) % 4);
      auto issue = [&](int k) {   // box k of this group into the next slot
        const int64_t i0 = ibeg + (int64_t)k * kItR;
        const int x = MIRROR ? (int)((int64_t)W - 1 - (i0 + d0 + 62)) - sh : (int)(i0 + d0) - sh;
        const uint32_t slot = nissue % kItNB;
        if (lane == 0) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          it_box(ring + slot * (kItR * kItX * 4), tmap, x, (int)i0, bar0 + 8 * slot);
        }
        ++nissue;
      };
      for (int k = 0; k < kItNB - 1 && k < nbox; ++k) issue(k);
      for (int k = 0; k < nbox; ++k) {
        const uint32_t slot = nuse % kItNB;
        it_wait(bar0 + 8 * slot, (nuse / kItNB) & 1u);
        const int64_t i0 = ibeg + (int64_t)k * kItR;
        const uint32_t base = ring + slot * (kItR * kItX * 4);
        int32_t g[kItR];
#pragma unroll
        for (int u = 0; u < kItR; ++u) {
          const int c = MIRROR ? (62 - u - lane + sh) : (u + lane + sh);
          asm volatile("ld.shared.b32 %0, [%1];" : "=r"(g[u]) : "r"(base + (uint32_t)(u * kItX + c) * 4u));
        }
        __syncwarp();   // every lane has read the slot: it can be refilled
        ++nuse;
        if (k + kItNB - 1 < nbox) issue(k + kItNB - 1);
        const bool full = live && i0 >= ia && i0 + kItR <= ib;
        // every lane's 32 cells inside the table and off row 0 / column 0: f reduces to
        // max(cell, UL) + c (CellDiagMaxPlus::f without its boundary selects: two ops per cell on
        // the chain instead of the int64 row / column tests)
        if (__all_sync(0xffffffffu, full && i0 >= 1 && i0 + d0 + p.col0 >= 1)) {
          const int32_t c = p.param_c;
#pragma unroll
          for (int u = 0; u < kItR; ++u) v = max(g[u], v) + c;
        } else {
#pragma unroll
          for (int u = 0; u < kItR; ++u) {
            const int64_t i = i0 + u;
            if (full || (live && i >= ia && i < ib)) {
              int32_t o;
              v = F::f(v, v, v, v, 0, 0, g[u], i, (int)(i + d) + p.col0, p.param_c, o);
            }
          }
        }
      }
      // the chain ends in the last row (ib == H) or the last column (j == W-1)
      if (live && ib > ia) {
        const int64_t jl = ib - 1 + d;
        const int64_t jg = MIRROR ? (int64_t)W - 1 - jl : jl;
        if (ib == H && p.last_row != nullptr) static_cast<T*>(p.last_row)[jg] = v;
        if (jl == W - 1 && p.last_col != nullptr) static_cast<T*>(p.last_col)[ib - 1] = v;
      }
    }
  }
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link needed)
static PFN_cuTensorMapEncodeTiled_v12000 it_encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (fn == nullptr) {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
  }
  return fn;
}

// DIAG_MAXPLUS / ANTIDIAG_MAXPLUS without TABLE: the TMA kernel when the grid qualifies
// (16-byte aligned base, pitch % 4 == 0, an encoder); returns cudaErrorNotSupported otherwise.
cudaError_t launch_invl_tma(const FillParams& p, bool mirror, int sms, cudaStream_t s) {
  if (p.table != nullptr || (reinterpret_cast<uintptr_t>(p.grid) & 15) || (p.grid_pitch % 4) || p.cols <= 0 ||
      p.rows <= 0)
    return cudaErrorNotSupported;
  PFN_cuTensorMapEncodeTiled_v12000 enc = it_encode_fn();
  if (enc == nullptr) return cudaErrorNotSupported;
  CUtensorMap tm;
  memset(&tm, 0, sizeof(tm));
  const cuuint64_t dims[2] = {(cuuint64_t)p.cols, (cuuint64_t)p.rows};
  const cuuint64_t strides[1] = {(cuuint64_t)p.grid_pitch * 4};
  const cuuint32_t box[2] = {(cuuint32_t)kItX, (cuuint32_t)kItR};
  const cuuint32_t estr[2] = {1, 1};
  if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_INT32, 2, const_cast<void*>(p.grid), dims, strides, box, estr,
          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return cudaErrorNotSupported;
  auto k = mirror ? invl_tma_kernel<true> : invl_tma_kernel<false>;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(invl_tma_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kItSmem);
    cudaFuncSetAttribute(invl_tma_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kItSmem);
    attr = true;
  }
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kItWarps * 32, kItSmem);
  const int64_t NG = (p.diag_hi - p.diag_lo + 31) / 32;
  const int64_t NP = (NG + 1) / 2;
  const int64_t want = (NP + kItWarps - 1) / kItWarps;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)sms * std::max(occ, 1)));
  FillParams pp = p;
  void* args[] = {&pp, &tm};
  return cudaLaunchKernel((const void*)k, dim3(grid), dim3(kItWarps * 32), args, kItSmem, s);
}

// func 4 DIAG_MAXPLUS (Inverted-L) and 8 ANTIDIAG_MAXPLUS (its mirror twin, the same cell on the
// mirrored grid, mirror = true)
cudaError_t launch_invl(int func, const FillParams& p, int grid, bool mirror, cudaStream_t s) {
  if (func != 4 && func != 8) return cudaErrorInvalidValue;
  return mirror ? launch_il<CellDiagMaxPlus, true>(p, grid, s) : launch_il<CellDiagMaxPlus, false>(p, grid, s);
}

}  // namespace lddp
