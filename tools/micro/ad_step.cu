// ad_step.cu -- microbenchmark of the adiag steady inner loop in isolation (development tool):
// one warp sweeps n columns of a lane-systolic LCS strip (R rows per lane, rows chained, lane
// lag E), with the column character from global memory (CMODE 0, prefetched one 8-step group
// ahead), from shared memory (1) or a register (2), and the top-row injection shuffle (INJ).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ad_step ad_step.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int R, int E, int CMODE, int INJ, int UNR>
__global__ void sweep(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a, int* out,
                      long long* cyc) {
  __shared__ uint8_t sb[1 << 15];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < n; i += blockDim.x) sb[i] = b[i];
  __syncthreads();
  int ar[R];
  for (int r = 0; r < R; ++r) ar[r] = a[(threadIdx.x * R + r) & 4095];
  int hist[R], fifo[E + 1], cc[8];
  for (int r = 0; r < R; ++r) hist[r] = 0;
  for (int d = 0; d <= E; ++d) fifo[d] = 0;
  for (int u = 0; u < 8; ++u) cc[u] = b[u];
  int topv = lane;
  long long t0 = clock64();
#pragma unroll 1
  for (int t = 0; t < n; t += 8 * UNR) {
#pragma unroll
    for (int q = 0; q < UNR; ++q) {
      int cn[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = (t + 8 * q + 8 + u - lane * E) & (n - 1);
        cn[u] = CMODE == 0 ? (int)b[c] : (CMODE == 1 ? (int)sb[c] : c & 3);
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        int U = fifo[E - 1], UL = fifo[E];
        int nw[R];
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int v = max(max(U, hist[r]), UL + (ar[r] == cc[u] ? 1 : 0));
          UL = hist[r];
          U = v;
          nw[r] = v;
        }
        int sv = nw[R - 1];
        if (INJ) {
          const int inj = __shfl_sync(0xffffffffu, topv, 8 * q + u);
          sv = (lane == 31) ? inj : sv;
        }
        const int rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
        for (int d = E; d > 0; --d) fifo[d] = fifo[d - 1];
        fifo[0] = rv;
#pragma unroll
        for (int r = 0; r < R; ++r) hist[r] = nw[r];
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) cc[u] = cn[u];
    }
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += hist[r];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc + fifo[0];
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int R, int E, int CMODE, int INJ, int UNR>
void run(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n, int blocks, int warps) {
  sweep<R, E, CMODE, INJ, UNR><<<blocks, 32 * warps>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[1];
  cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("R=%d E=%d CMODE=%d INJ=%d UNR=%d blocks=%d warps=%d: %.1f cycles/step (%.2f cells/clk/warp)\n", R, E,
         CMODE, INJ, UNR, blocks, warps, (double)h[0] / n, 32.0 * R * n / (double)h[0]);
}

int main() {
  const int n = 1 << 15;
  uint8_t *b, *a;
  int* out;
  long long* cyc;
  cudaMalloc(&b, n);
  cudaMalloc(&a, 4096);
  cudaMalloc(&out, 1 << 22);
  cudaMalloc(&cyc, 1 << 16);
  cudaMemset(b, 1, n);
  cudaMemset(a, 2, 4096);
  run<6, 2, 0, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 1, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 2, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 2, 0, 1>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 0, 1, 4>(b, a, out, cyc, n, 1, 1);
  run<6, 3, 0, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<2, 2, 0, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<4, 2, 0, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<8, 2, 0, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 0, 1, 1>(b, a, out, cyc, n, 148, 4);
  run<6, 2, 1, 1, 1>(b, a, out, cyc, n, 148, 4);
  run<6, 2, 0, 1, 1>(b, a, out, cyc, n, 148, 8);
  return 0;
}
