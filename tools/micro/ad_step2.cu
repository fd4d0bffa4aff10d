// ad_step2.cu -- LCS lane-systolic step variants (development tool).
//  ADD 0: compiler's UL + 1 (VIADD); 1: IMAD with a run-time one (FMA pipe)
//  CC  0: LDG one group ahead; 1: LDS one group ahead; 2: constant; 3: forwarded by a 2nd SHFL
//        (lane 31 injects the column character lane 0 needs, read from smem by broadcast)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ int imad1(int x, int one) {
  int r;
  asm("mad.lo.s32 %0, %1, %2, %2;" : "=r"(r) : "r"(x), "r"(one));
  return r;
}

template <int R, int E, int ADD, int CC>
__global__ void sweep(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a, int* out,
                      long long* cyc, int one) {
  __shared__ uint8_t sb[1 << 15];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < n; i += blockDim.x) sb[i] = b[i];
  __syncthreads();
  int ar[R];
  for (int r = 0; r < R; ++r) ar[r] = a[(threadIdx.x * R + r) & 4095];
  int hist[R], fifo[E + 1], cc[8], cf[E + 1];
  for (int r = 0; r < R; ++r) hist[r] = 0;
  for (int d = 0; d <= E; ++d) { fifo[d] = 0; cf[d] = 0; }
  for (int u = 0; u < 8; ++u) cc[u] = b[u];
  int topv = lane;
  long long t0 = clock64();
#pragma unroll 1
  for (int t = 0; t < n; t += 8) {
    int cn[8];
    if (CC < 3) {
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = (t + 8 + u - lane * E) & (n - 1);
        cn[u] = CC == 0 ? (int)b[c] : (CC == 1 ? (int)sb[c] : c & 3);
      }
    } else {
#pragma unroll
      for (int u = 0; u < 8; ++u) cn[u] = sb[(t + 8 + u + E) & (n - 1)];   // broadcast: lane 0's future column
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      int U = fifo[E - 1], UL = fifo[E];
      const int c_u = (CC == 3) ? cf[E - 1] : cc[u];
      int nw[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int ulp = ADD ? imad1(UL, one) : UL + 1;
        const int t2 = (ar[r] == c_u) ? ulp : UL;
        const int v = max(max(U, hist[r]), t2);
        UL = hist[r];
        U = v;
        nw[r] = v;
      }
      const int inj = __shfl_sync(0xffffffffu, topv, u);
      const int sv = (lane == 31) ? inj : nw[R - 1];
      const int rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
      for (int d = E; d > 0; --d) fifo[d] = fifo[d - 1];
      fifo[0] = rv;
      if (CC == 3) {
        const int sc = (lane == 31) ? cc[u] : c_u;
        const int rc = __shfl_sync(0xffffffffu, sc, (lane + 31) & 31);
#pragma unroll
        for (int d = E; d > 0; --d) cf[d] = cf[d - 1];
        cf[0] = rc;
      }
#pragma unroll
      for (int r = 0; r < R; ++r) hist[r] = nw[r];
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) cc[u] = cn[u];
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += hist[r];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc + fifo[0] + cf[0];
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int R, int E, int ADD, int CC>
void run(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n, int blocks, int warps) {
  sweep<R, E, ADD, CC><<<blocks, 32 * warps>>>(b, n, a, out, cyc, 1);
  cudaDeviceSynchronize();
  long long h[1];
  cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("R=%d E=%d ADD=%d CC=%d blocks=%d warps=%d: %.1f cycles/step (%.2f cells/clk/warp)\n", R, E, ADD, CC,
         blocks, warps, (double)h[0] / n, 32.0 * R * n / (double)h[0]);
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
  run<6, 2, 0, 2>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 1, 2>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 1, 0>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 1, 3>(b, a, out, cyc, n, 1, 1);
  run<6, 3, 1, 2>(b, a, out, cyc, n, 1, 1);
  run<6, 3, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<6, 3, 1, 3>(b, a, out, cyc, n, 1, 1);
  run<8, 2, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<8, 2, 1, 3>(b, a, out, cyc, n, 1, 1);
  run<4, 2, 1, 1>(b, a, out, cyc, n, 1, 1);
  run<4, 2, 1, 3>(b, a, out, cyc, n, 1, 1);
  run<6, 2, 1, 1>(b, a, out, cyc, n, 148, 4);
  run<6, 2, 1, 3>(b, a, out, cyc, n, 148, 4);
  return 0;
}
