// fsstep.cu -- cycles per step of the lane-systolic FS body (one row per lane, one warp per SM
// sub-partition, private rows, no links).  Development tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 --fmad=false -o fsstep fsstep.cu && ./fsstep
// MODE 0: full body (LDS.U8 + I2F input, STS.U8 output, rotate SHFL, E)
// MODE 1: no input load (constant 100.f)
// MODE 2: no SHFL (U* from the lane's own history)
// MODE 3: input as float from smem (LDS.32, no I2F)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int E, int MODE>
__global__ void __launch_bounds__(128, 1) fs(int n, int* out, long long* cyc) {
  __shared__ uint8_t inr[4][32][128];
  __shared__ float inf[4][32][64];
  __shared__ uint8_t outr[4][32][64];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 4 * 32 * 128; i += blockDim.x) { (&inr[0][0][0])[i] = (uint8_t)(i * 7); if (i < 4 * 32 * 64) (&inf[0][0][0])[i] = (float)(i & 255); }
  __syncthreads();
  constexpr int D = 2 + E;
  float fifo[E + 3];
  for (int d = 0; d < E + 3; ++d) fifo[d] = 0.f;
  float eL = 0.f;
  float inq[16];
  for (int u = 0; u < 16; ++u) inq[u] = (float)inr[w][lane][(u - D * lane) & 127];
  long long t0 = clock64();
  for (int t = 0; t < n; t += 16) {
    float inn[16];
    if (MODE == 4) {
#pragma unroll
      for (int u = 0; u < 16; ++u) inn[u] = (float)inr[w][lane][(t + 16 + u - D * lane) & 127];
    }
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      const int tau = t + u;
      const int c = tau - D * lane;
      float in;
      if (MODE == 4) in = inq[u];
      else if (MODE == 1) in = 100.f;
      else if (MODE == 3) in = inf[w][lane][c & 63];
      else in = (float)inr[w][lane][c & 127];
      const float UR = MODE == 2 ? eL : fifo[E], U = MODE == 2 ? fifo[0] : fifo[E + 1], UL = fifo[E + 2];
      float v = __fadd_rn(in, __fmul_rn(UL, 0.0625f));
      v = __fadd_rn(v, __fmul_rn(U, 0.3125f));
      v = __fadd_rn(v, __fmul_rn(UR, 0.1875f));
      v = __fadd_rn(v, __fmul_rn(eL, 0.4375f));
      const bool hi = v >= 128.0f;
      outr[w][lane][c & 63] = hi ? 255 : 0;
      float e = hi ? __fsub_rn(v, 255.0f) : v;
      e = ((unsigned)c < (unsigned)n) ? e : 0.0f;
      eL = e;
      float rv = e;
      if (MODE != 2) rv = __shfl_sync(0xffffffffu, e, (lane + 31) & 31);
#pragma unroll
      for (int d = E + 2; d > 0; --d) fifo[d] = fifo[d - 1];
      fifo[0] = rv;
    }
    if (MODE == 4) {
#pragma unroll
      for (int u = 0; u < 16; ++u) inq[u] = inn[u];
    }
  }
  long long t1 = clock64();
  out[blockIdx.x * 128 + threadIdx.x] = (int)(eL + fifo[0]) + outr[w][lane][lane];
  if (lane == 0) cyc[blockIdx.x * 4 + w] = t1 - t0;
}

template <int E, int MODE>
void run(int* out, long long* cyc, int n) {
  fs<E, MODE><<<148, 128>>>(n, out, cyc);
  cudaDeviceSynchronize();
  fs<E, MODE><<<148, 128>>>(n, out, cyc);
  cudaDeviceSynchronize();
  long long h[148 * 4];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148 * 4; ++i) s += (double)h[i];
  s /= 148 * 4;
  printf("E=%d MODE=%d: %.1f cycles/step\n", E, MODE, s / n);
}


// Two rows per lane, skew 2 inside the lane (row 1 two columns behind row 0): two independent
// pixel chains per step; row 1 takes U / UR / UL from row 0's error history.
template <int E>
__global__ void __launch_bounds__(128, 1) fs2(int n, int* out, long long* cyc) {
  __shared__ uint8_t inr[4][32][2][128];
  __shared__ uint8_t outr[4][32][2][64];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 4 * 32 * 2 * 128; i += blockDim.x) (&inr[0][0][0][0])[i] = (uint8_t)(i * 7);
  __syncthreads();
  constexpr int D = 4 + E;   // lane lag: 2 rows x 2 columns + E
  float fifo[E + 3];
  for (int d = 0; d < E + 3; ++d) fifo[d] = 0.f;
  float h0[3] = {0.f, 0.f, 0.f};   // row 0 error at steps t-1, t-2, t-3
  float eL1 = 0.f;
  float inq0[16], inq1[16];
  for (int u = 0; u < 16; ++u) { inq0[u] = (float)inr[w][lane][0][(u - D * lane) & 127]; inq1[u] = (float)inr[w][lane][1][(u - 2 - D * lane) & 127]; }
  long long t0 = clock64();
  for (int t = 0; t < n; t += 16) {
    float inn0[16], inn1[16];
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      inn0[u] = __fsub_rn(__uint_as_float(0x4B000000u | inr[w][lane][0][(t + 16 + u - D * lane) & 127]), 8388608.0f);
      inn1[u] = __fsub_rn(__uint_as_float(0x4B000000u | inr[w][lane][1][(t + 14 + u - D * lane) & 127]), 8388608.0f);
    }
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      const int tau = t + u;
      const int c0 = tau - D * lane, c1 = c0 - 2;
      // row 0: neighbours from the lane above (fifo)
      float v = __fadd_rn(inq0[u], __fmul_rn(fifo[E + 2], 0.0625f));
      v = __fadd_rn(v, __fmul_rn(fifo[E + 1], 0.3125f));
      v = __fadd_rn(v, __fmul_rn(fifo[E], 0.1875f));
      v = __fadd_rn(v, __fmul_rn(h0[0], 0.4375f));
      bool hi = v >= 128.0f;
      outr[w][lane][0][c0 & 63] = hi ? 255 : 0;
      float e0 = hi ? __fsub_rn(v, 255.0f) : v;
      e0 = ((unsigned)c0 < (unsigned)n) ? e0 : 0.0f;
      // row 1 (column c0 - 2): UR = row 0 at c0-1 (step t-1), U = c0-2 (t-2), UL = c0-3 (t-3)
      float x = __fadd_rn(inq1[u], __fmul_rn(h0[2], 0.0625f));
      x = __fadd_rn(x, __fmul_rn(h0[1], 0.3125f));
      x = __fadd_rn(x, __fmul_rn(h0[0], 0.1875f));
      x = __fadd_rn(x, __fmul_rn(eL1, 0.4375f));
      hi = x >= 128.0f;
      outr[w][lane][1][c1 & 63] = hi ? 255 : 0;
      float e1 = hi ? __fsub_rn(x, 255.0f) : x;
      e1 = ((unsigned)c1 < (unsigned)n) ? e1 : 0.0f;
      eL1 = e1;
      h0[2] = h0[1]; h0[1] = h0[0]; h0[0] = e0;
      const float rv = __shfl_sync(0xffffffffu, e1, (lane + 31) & 31);
#pragma unroll
      for (int d = E + 2; d > 0; --d) fifo[d] = fifo[d - 1];
      fifo[0] = rv;
    }
#pragma unroll
    for (int u = 0; u < 16; ++u) { inq0[u] = inn0[u]; inq1[u] = inn1[u]; }
  }
  long long t1 = clock64();
  out[blockIdx.x * 128 + threadIdx.x] = (int)(eL1 + fifo[0] + h0[0]) + outr[w][lane][0][lane] + outr[w][lane][1][lane];
  if (lane == 0) cyc[blockIdx.x * 4 + w] = t1 - t0;
}

template <int E>
void run2(int* out, long long* cyc, int n) {
  fs2<E><<<148, 128>>>(n, out, cyc);
  cudaDeviceSynchronize();
  fs2<E><<<148, 128>>>(n, out, cyc);
  cudaDeviceSynchronize();
  long long h[148 * 4];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148 * 4; ++i) s += (double)h[i];
  s /= 148 * 4;
  printf("R=2 E=%d: %.1f cycles/step (2 pixels)\n", E, s / n);
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 128 * 4);
  cudaMalloc(&cyc, 148 * 4 * 8);
  const int n = 1 << 14;
  run<1, 0>(out, cyc, n);
  run<1, 1>(out, cyc, n);
  run<1, 2>(out, cyc, n);
  run<1, 3>(out, cyc, n);
  run<1, 4>(out, cyc, n);
  run2<1>(out, cyc, n);
  run2<0>(out, cyc, n);
  run<2, 0>(out, cyc, n);
  run<3, 0>(out, cyc, n);
  return 0;
}
