// lat2.cu -- dependent latency of one cell of each compiled f along its critical dependency
// (one warp, a chain of N cells where each cell's input is the previous cell's output), on the
// B200's SM clock.  These are the constants of the span roofline (T_span =
// longest dependency path x per-cell latency), printed as JSON.  Development / measurement tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 --fmad=false -o lat2 lat2.cu && ./lat2
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k(const int* __restrict__ g, int n, int* out, long long* cyc) {
  const int lane = threadIdx.x;
  int x = g[lane], y = g[lane + 32], z = g[lane + 64];
  const int one = g[96] | 1;
  long long t0, t1;
  // LCS cell along U (or L): v = max3(U, L, UL + m): the chain runs through VIMNMX3
  t0 = clock64();
  for (int i = 0; i < n; ++i) x = max(max(x, y), z + (i & one));
  t1 = clock64();
  if (lane == 0) cyc[0] = t1 - t0;
  // Levenshtein cell: v = min3(U + 1, L + 1, UL + [a != b]) -> chain through an add and a min3
  int w = x;
  t0 = clock64();
  for (int i = 0; i < n; ++i) w = min(min(w + one, y + one), z + (i & 1));
  t1 = clock64();
  if (lane == 0) cyc[1] = t1 - t0;
  // DTW cell: D = |x - y| + min3(U, L, UL): chain through FMNMX3 and FADD
  float fu = (float)x, fl = (float)y, ful = (float)z, d = (float)(lane + 1);
  t0 = clock64();
  for (int i = 0; i < n; ++i) fu = d + fminf(fminf(fu, fl), ful);
  t1 = clock64();
  if (lane == 0) cyc[2] = t1 - t0;
  // Floyd-Steinberg pull form along L: v = in + 1/16 UL + 5/16 U + 3/16 UR + 7/16 L; threshold;
  // error = v - out (no FMA contraction, the kernel's operation order)
  float eL = 0.f, base = (float)(lane & 127);
  t0 = clock64();
  for (int i = 0; i < n; ++i) {
    float v = __fadd_rn(base, __fmul_rn(fu, 0.0625f));
    v = __fadd_rn(v, __fmul_rn(fl, 0.3125f));
    v = __fadd_rn(v, __fmul_rn(ful, 0.1875f));
    v = __fadd_rn(v, __fmul_rn(eL, 0.4375f));
    eL = v >= 128.0f ? __fsub_rn(v, 255.0f) : v;
  }
  t1 = clock64();
  if (lane == 0) cyc[3] = t1 - t0;
  // min-path row chain (previous-row category, one column): f = c + min3(UL, U, UR)
  int u = x;
  t0 = clock64();
  for (int i = 0; i < n; ++i) u = (i & 1023) + min(min(u, y), z);
  t1 = clock64();
  if (lane == 0) cyc[4] = t1 - t0;
  // rotate SHFL (lane k-1 -> k): the lane-to-lane hop of every lane-systolic kernel
  int s = x;
  t0 = clock64();
  for (int i = 0; i < n; ++i) s = __shfl_sync(0xffffffffu, s, (lane + 31) & 31) + 1;
  t1 = clock64();
  if (lane == 0) cyc[5] = t1 - t0;
  out[lane] = x + w + u + s + (int)(fu + eL);
}

int main() {
  int *g, *out;
  long long* cyc;
  cudaMalloc(&g, 1024 * 4);
  cudaMalloc(&out, 4096);
  cudaMalloc(&cyc, 64 * 8);
  int h[1024];
  for (int i = 0; i < 1024; ++i) h[i] = (i * 7 + 1) & 1023;
  cudaMemcpy(g, h, sizeof h, cudaMemcpyHostToDevice);
  const int n = 1 << 16;
  k<<<1, 32>>>(g, n, out, cyc);   // warm-up
  k<<<1, 32>>>(g, n, out, cyc);
  cudaDeviceSynchronize();
  long long c[8];
  cudaMemcpy(c, cyc, sizeof c, cudaMemcpyDeviceToHost);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("{\"lcs_cell\": %.2f, \"levenshtein_cell\": %.2f, \"dtw_cell\": %.2f, \"fs_cell\": %.2f, "
         "\"minpath_row\": %.2f, \"shfl_hop\": %.2f, \"unit\": \"SM cycles per dependent cell\", "
         "\"how\": \"tools/micro/lat2.cu: one warp, 65536-cell dependent chain, clock64\"}\n",
         (double)c[0] / n, (double)c[1] / n, (double)c[2] / n, (double)c[3] / n, (double)c[4] / n,
         (double)c[5] / n);
  return 0;
}
