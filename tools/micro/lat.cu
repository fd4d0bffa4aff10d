// lat.cu -- dependent-latency microbenchmarks on one warp (development tool): VIMNMX3 chain,
// the LCS cell chain, SHFL chain, L1-hit LDG chain, LDS chain.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__global__ void k(const int* __restrict__ g, int n, int* out, long long* cyc) {
  __shared__ int sm[1024];
  const int lane = threadIdx.x;
  for (int i = lane; i < 1024; i += 32) sm[i] = (i + 1) & 1023;
  __syncwarp();
  int x = lane, y = lane + 1, z = lane + 2;
  long long t0, t1;
  // 1. VIMNMX3 chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { x = max(max(x, y), z + i); }
  t1 = clock64(); if (lane == 0) cyc[0] = t1 - t0;
  // 2. LCS cell chain (U -> v), predicate from a loop-invariant compare
  int a = g[lane], b = g[lane + 1];
  t0 = clock64();
  for (int i = 0; i < n; ++i) { x = max(max(x, y), z + (a == (b ^ i) ? 1 : 0)); }
  t1 = clock64(); if (lane == 0) cyc[1] = t1 - t0;
  // 3. SHFL chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { x = __shfl_sync(0xffffffffu, x, (lane + 31) & 31) + 1; }
  t1 = clock64(); if (lane == 0) cyc[2] = t1 - t0;
  // 4. LDG chain (L1 hit)
  int p = lane;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { p = g[p & 1023]; }
  t1 = clock64(); if (lane == 0) cyc[3] = t1 - t0;
  // 5. LDS chain
  int q = lane;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { q = sm[q & 1023]; }
  t1 = clock64(); if (lane == 0) cyc[4] = t1 - t0;
  // 6. FADD+FMNMX chain
  float fx = lane, fy = 1, fz = 2;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { fx = fabsf(fy - fz) + fminf(fminf(fx, fy), fz); }
  t1 = clock64(); if (lane == 0) cyc[5] = t1 - t0;
  // 7. SEL + SHFL chain (the rotate with lane-31 injection)
  t0 = clock64();
  for (int i = 0; i < n; ++i) { int s = lane == 31 ? y : x; x = __shfl_sync(0xffffffffu, s, (lane + 31) & 31); }
  t1 = clock64(); if (lane == 0) cyc[6] = t1 - t0;
  out[lane] = x + y + z + p + q + (int)fx;
}
int main() {
  int *g, *out; long long* cyc;
  cudaMalloc(&g, 4096 * 4); cudaMalloc(&out, 4096); cudaMalloc(&cyc, 64 * 8);
  int h[1024]; for (int i = 0; i < 1024; ++i) h[i] = (i + 1) & 1023;
  cudaMemcpy(g, h, 4096, cudaMemcpyHostToDevice);
  const int n = 4096;
  k<<<1, 32>>>(g, n, out, cyc);
  cudaDeviceSynchronize();
  long long c[8]; cudaMemcpy(c, cyc, 64, cudaMemcpyDeviceToHost);
  const char* names[] = {"VIMNMX3 chain", "LCS cell chain", "SHFL(+1) chain", "LDG L1 chain", "LDS chain", "DTW cell chain", "SEL+SHFL chain"};
  for (int i = 0; i < 7; ++i) printf("%-16s %.1f cycles/iter\n", names[i], (double)c[i] / n);
  return 0;
}
