// rowstep.cu -- cycles per row of the prev-row column-block loop (one warp per SM
// sub-partition, no memory stream): where do ~150 cycles per row come from?  Development tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o rowstep rowstep.cu && ./rowstep
// MODE 0: LDS.128 costs + SHFL up/down + VP cells   (the prevrow_cb body)
// MODE 1: no LDS (costs in registers)
// MODE 2: SHFL up only (UR from own register)
// MODE 3: no SHFL (UL/UR from own registers)
// MODE 4: as 0 with the LDS one row ahead in a second register set
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int VP, int MODE, int RING = 16>
__global__ void __launch_bounds__(128, 1) rows(int n, int* out, long long* cyc, const int* __restrict__ gsrc) {
  __shared__ __align__(16) int ring[4][8][32 * VP];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 4 * 8 * 32 * VP; i += blockDim.x) (&ring[0][0][0])[i] = i & 1023;
  __syncthreads();
  int cur[VP], gk[VP], gn[VP];
  for (int v = 0; v < VP; ++v) { cur[v] = lane + v; gk[v] = v; gn[v] = v; }
  // MODE 5 / 6: + one 16-byte cp.async per lane per row from global (6: every 4th row commits)
  extern __shared__ __align__(16) int cdyn[];
  const uint32_t cbase = (uint32_t)__cvta_generic_to_shared(cdyn + (size_t)w * RING * 128 + lane * 4);
  long long t0 = clock64();
  for (int r = 0; r < n; ++r) {
    if (MODE >= 5) {
      const int* src = gsrc + ((size_t)(r & 4095) * 32768 + blockIdx.x * 128 + threadIdx.x * 4);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(cbase + (r & (RING - 1)) * 512), "l"(src) : "memory");
      if (MODE == 5 || (r & 3) == 3) {
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group %0;" ::"n"(RING - 2) : "memory");
      }
    }
    int g[VP];
    if (MODE == 1 || MODE >= 5) {
#pragma unroll
      for (int v = 0; v < VP; ++v) g[v] = gk[v] + (r & 1);
    } else if (MODE == 4) {
#pragma unroll
      for (int v = 0; v < VP; ++v) g[v] = gn[v];
      const int4* src = reinterpret_cast<const int4*>(&ring[w][(r + 1) & 7][lane * VP]);
#pragma unroll
      for (int s = 0; s < VP / 4; ++s) { int4 t = src[s]; gn[4 * s] = t.x; gn[4 * s + 1] = t.y; gn[4 * s + 2] = t.z; gn[4 * s + 3] = t.w; }
    } else {
      const int4* src = reinterpret_cast<const int4*>(&ring[w][r & 7][lane * VP]);
#pragma unroll
      for (int s = 0; s < VP / 4; ++s) { int4 t = src[s]; g[4 * s] = t.x; g[4 * s + 1] = t.y; g[4 * s + 2] = t.z; g[4 * s + 3] = t.w; }
    }
    int lv, rv;
    if (MODE == 3) { lv = cur[VP - 1]; rv = cur[0]; }
    else {
      lv = __shfl_up_sync(0xffffffffu, cur[VP - 1], 1);
      rv = (MODE == 2) ? cur[0] : __shfl_down_sync(0xffffffffu, cur[0], 1);
    }
    int nw[VP];
#pragma unroll
    for (int v = 0; v < VP; ++v) {
      const int UL = v > 0 ? cur[v - 1] : lv;
      const int UR = v < VP - 1 ? cur[v + 1] : rv;
      nw[v] = g[v] + __vimin3_s32(UL, cur[v], UR);
    }
#pragma unroll
    for (int v = 0; v < VP; ++v) cur[v] = nw[v];
  }
  long long t1 = clock64();
  int acc = 0;
  for (int v = 0; v < VP; ++v) acc += cur[v];
  out[blockIdx.x * 128 + threadIdx.x] = acc;
  if (lane == 0) cyc[blockIdx.x * 4 + w] = t1 - t0;
}

template <int VP, int MODE, int RING = 16>
void run(int* out, long long* cyc, int n, const int* g) {
  const int dyn = 4 * RING * 512;
  cudaFuncSetAttribute(rows<VP, MODE, RING>, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn);
  rows<VP, MODE, RING><<<148, 128, dyn>>>(n, out, cyc, g);
  cudaDeviceSynchronize();
  rows<VP, MODE, RING><<<148, 128, dyn>>>(n, out, cyc, g);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[148 * 4];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148 * 4; ++i) s += (double)h[i];
  s /= 148 * 4;
  printf("VP=%d MODE=%d RING=%d: %.1f cycles/row (%s)\n", VP, MODE, RING, s / n, cudaGetErrorString(e));
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 128 * 4);
  cudaMalloc(&cyc, 148 * 4 * 8);
  const int n = 1 << 14;
  int* g;
  cudaMalloc(&g, (size_t)4096 * 32768 * 4);
  run<4, 0>(out, cyc, n, g);
  run<4, 1>(out, cyc, n, g);
  run<4, 4>(out, cyc, n, g);
  run<4, 5>(out, cyc, n, g);
  run<4, 5, 32>(out, cyc, n, g);
  run<4, 5, 64>(out, cyc, n, g);
  return 0;
}
