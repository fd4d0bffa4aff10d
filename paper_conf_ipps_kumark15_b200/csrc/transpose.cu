// transpose.cu -- tiled out-of-place transpose of a 32-bit grid, the data movement behind the
// Vertical category: "Vertical is the transpose of Horizontal" [L111] (Table I [L109-L113]).
// 32 x 32 tiles through shared memory (one padding column: no bank conflicts), coalesced
// 128-byte row segments on both sides.  HBM bound: 8 bytes per cell.
#include <cstdint>
#include <cuda_runtime.h>

namespace lddp {

__global__ void __launch_bounds__(256) transpose_i32_kernel(const int32_t* __restrict__ src, int64_t spitch,
                                                            int32_t* __restrict__ dst, int64_t dpitch,
                                                            int64_t rows, int64_t cols) {
  __shared__ int32_t tile[32][33];
  const int64_t r0 = (int64_t)blockIdx.y * 32, c0 = (int64_t)blockIdx.x * 32;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;   // 8 rows of 32 threads
#pragma unroll
  for (int k = 0; k < 32; k += 8) {
    const int64_t r = r0 + ty + k, c = c0 + tx;
    if (r < rows && c < cols) tile[ty + k][tx] = __ldcs(src + r * spitch + c);
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < 32; k += 8) {
    const int64_t c = c0 + ty + k, r = r0 + tx;   // dst row c, column r
    if (r < rows && c < cols) dst[c * dpitch + r] = tile[tx][ty + k];
  }
}

// dst (cols x rows, pitch dpitch) = transpose of src (rows x cols, pitch spitch); elements.
cudaError_t launch_transpose_i32(const int32_t* src, int64_t spitch, int32_t* dst, int64_t dpitch, int64_t rows,
                                 int64_t cols, cudaStream_t s) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  const int64_t gx = (cols + 31) / 32, gy = (rows + 31) / 32;
  if (gy > 65535) return cudaErrorInvalidValue;
  transpose_i32_kernel<<<dim3((unsigned)gx, (unsigned)gy), 256, 0, s>>>(src, spitch, dst, dpitch, rows, cols);
  return cudaGetLastError();
}

}  // namespace lddp
