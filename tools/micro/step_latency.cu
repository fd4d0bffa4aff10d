// step_latency.cu -- microbenchmark of one warp sweeping a lane-systolic LCS strip (no links,
// no flags): cycles per step for several exchange styles.  Development tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o step_latency step_latency.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int R, int MODE>
__global__ void sweep(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a, int* out,
                      long long* cyc) {
  // MODE 0: value + char via 2 SHFL per step (rows chained, lag 2)
  // MODE 1: value via SHFL, char from smem per lane (LDS)
  // MODE 2: value + char packed in 1 SHFL
  __shared__ uint8_t sb[1 << 15];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < n; i += blockDim.x) sb[i] = b[i];
  __syncthreads();
  int ar[R];
  for (int r = 0; r < R; ++r) ar[r] = a[lane * R + r];
  int hist[R], f0 = 0, f1 = 0, f2 = 0, c0 = 0, c1 = 0;
  for (int r = 0; r < R; ++r) hist[r] = 0;
  long long t0 = clock64();
  for (int t = 0; t < n; t += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int tt = t + u;
      int cc;
      if (MODE == 1) cc = sb[(tt - 2 * lane) & 0x7fff];
      else cc = c1;
      int U = f1, UL = f2;
      int nw[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int L = hist[r];
        const int v = max(max(U, L), UL + (ar[r] == cc ? 1 : 0));
        UL = hist[r];
        U = v;
        nw[r] = v;
      }
      int sv = nw[R - 1], rv, rc;
      if (MODE == 2) {
        const int pk = (sv << 8) | (lane == 0 ? sb[tt & 0x7fff] : cc);
        const int rp = __shfl_sync(0xffffffffu, pk, (lane + 31) & 31);
        rv = rp >> 8;
        rc = rp & 0xff;
      } else {
        rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
        rc = (MODE == 0) ? __shfl_sync(0xffffffffu, lane == 0 ? (int)sb[tt & 0x7fff] : cc, (lane + 31) & 31) : 0;
      }
      f2 = f1; f1 = f0; f0 = rv;
      c1 = c0; c0 = rc;
#pragma unroll
      for (int r = 0; r < R; ++r) hist[r] = nw[r];
    }
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += hist[r];
  out[blockIdx.x * 32 + lane] = acc + f0 + c0;
  if (lane == 0) cyc[blockIdx.x] = t1 - t0;
}

// SIG = 1: lane row r processes column t - k*D - r; rows independent within a step.
// Column char rides down the rows in a register shift; row 0 gets value + char from the lane
// above through SHFL (two words) or the char from smem (CMODE 1).
template <int R, int E, int CMODE>
__global__ void sweep_skew(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a, int* out,
                           long long* cyc) {
  __shared__ uint8_t sb[1 << 15];
  const int lane = threadIdx.x & 31;
  constexpr int D = R + E;
  for (int i = threadIdx.x; i < n; i += blockDim.x) sb[i] = b[i];
  __syncthreads();
  int ar[R];
  for (int r = 0; r < R; ++r) ar[r] = a[lane * R + r];
  int h1[R], h2[R], hc[R];      // value at t-1, t-2; char at t-1
  int fv[E + 2], fc[E + 1];
  for (int r = 0; r < R; ++r) { h1[r] = 0; h2[r] = 0; hc[r] = 0; }
  for (int d = 0; d < E + 2; ++d) fv[d] = 0;
  for (int d = 0; d < E + 1; ++d) fc[d] = 0;
  long long t0 = clock64();
  for (int t = 0; t < n; t += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int tt = t + u;
      int nw[R], nc[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        int U, UL, cc;
        if (r == 0) {
          U = fv[E]; UL = fv[E + 1];
          cc = (CMODE == 1) ? (int)sb[(tt - lane * D) & 0x7fff] : fc[E];
        } else {
          U = h1[r - 1]; UL = h2[r - 1]; cc = hc[r - 1];
        }
        const int L = h1[r];
        nw[r] = max(max(U, L), UL + (ar[r] == cc ? 1 : 0));
        nc[r] = cc;
      }
      const int sv = nw[R - 1];
      const int rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
      int rc = 0;
      if (CMODE == 0) rc = __shfl_sync(0xffffffffu, lane == 0 ? (int)sb[tt & 0x7fff] : nc[R - 1], (lane + 31) & 31);
#pragma unroll
      for (int d = E + 1; d > 0; --d) fv[d] = fv[d - 1];
      fv[0] = rv;
#pragma unroll
      for (int d = E; d > 0; --d) fc[d] = fc[d - 1];
      fc[0] = rc;
#pragma unroll
      for (int r = 0; r < R; ++r) { h2[r] = h1[r]; h1[r] = nw[r]; hc[r] = nc[r]; }
    }
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += h1[r] + hc[r];
  out[blockIdx.x * 32 + lane] = acc + fv[0] + fc[0];
  if (lane == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int R, int E, int CMODE>
void run_skew(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n) {
  sweep_skew<R, E, CMODE><<<1, 32>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[1];
  cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("SKEW R=%d E=%d CMODE=%d: %.1f cycles/step (%.2f cells/cycle/warp)\n", R, E, CMODE,
         (double)h[0] / n, 32.0 * R * n / (double)h[0]);
}

template <int R, int MODE>
void run(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n, int blocks, int warps) {
  sweep<R, MODE><<<blocks, 32 * warps>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[1];
  cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("R=%d MODE=%d blocks=%d warps/blk=%d: %.1f cycles/step (%.2f cells/cycle/warp)\n", R, MODE, blocks,
         warps, (double)h[0] / n, 32.0 * R * n / (double)h[0]);
}

int main() {
  const int n = 1 << 15;
  uint8_t *b, *a;
  int* out;
  long long* cyc;
  cudaMalloc(&b, n);
  cudaMalloc(&a, 4096);
  cudaMalloc(&out, 1 << 20);
  cudaMalloc(&cyc, 1 << 16);
  cudaMemset(b, 1, n);
  cudaMemset(a, 2, 4096);
  run_skew<2, 1, 0>(b, a, out, cyc, n);
  run_skew<4, 1, 0>(b, a, out, cyc, n);
  run_skew<4, 2, 0>(b, a, out, cyc, n);
  run_skew<4, 1, 1>(b, a, out, cyc, n);
  run_skew<8, 1, 0>(b, a, out, cyc, n);
  run_skew<8, 2, 0>(b, a, out, cyc, n);
  run_skew<8, 1, 1>(b, a, out, cyc, n);
  run_skew<16, 1, 0>(b, a, out, cyc, n);
  run_skew<16, 1, 1>(b, a, out, cyc, n);
  run_skew<32, 1, 1>(b, a, out, cyc, n);
  for (int w : {1}) {
    run<4, 0>(b, a, out, cyc, n, 1, w);
    run<4, 1>(b, a, out, cyc, n, 1, w);
    run<4, 2>(b, a, out, cyc, n, 1, w);
    run<8, 0>(b, a, out, cyc, n, 1, w);
    run<8, 2>(b, a, out, cyc, n, 1, w);
    run<16, 2>(b, a, out, cyc, n, 1, w);
  }
  return 0;
}
