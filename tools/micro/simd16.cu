// simd16.cu -- one lane-systolic LCS step: 32-bit cells (the round-1 adiag body) against packed
// 16x2 cells (two rows per VIMNMX3.U16x2, match increments from one PRMT per row pair).  One warp
// per SM sub-partition sweeps its own private strip (no handoffs).  Development tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o simd16 simd16.cu && ./simd16
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t s) {
  uint32_t d;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(s));
  return d;
}
__device__ __forceinline__ uint32_t imad(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}
__device__ __forceinline__ uint32_t imadhi(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("mad.hi.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}

// MODE 0: 32-bit cells, R rows, match masks by PRMT of a packed per-code register (round 1)
// MODE 1: 16x2 cells, P pairs (rows p and P+p, the upper half one column behind)
// MODE 2: 16x2 cells, P pairs: lo halves = band A (lane k, rows kP..), hi halves = band B (rows
//         32P + kP..), band B 32E columns behind A: a 64-lane virtual warp, no packing
template <int P, int E, int MODE>
__global__ void __launch_bounds__(128, 1) sweep(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a,
                                                uint32_t* out, long long* cyc) {
  constexpr int R = 2 * P;
  constexpr int EL = MODE == 1 ? E + 1 : E;
  constexpr int DB = 32 * E;   // MODE 2: band B's column lag
  __shared__ __align__(16) uint32_t ring[4][256 + 8];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  // row codes of this lane (DNA: 0..3)
  int code[R];
  for (int r = 0; r < R; ++r) code[r] = a[(blockIdx.x * 128 + threadIdx.x) * R + r] & 3;
  // column ring: MODE 1 selectors, MODE 0 codes
  for (int i = lane; i < 264; i += 32) {
    const int c = i & 255;
    const int c0 = b[c] & 3, c1 = b[(c + (MODE == 2 ? 256 - DB : 255)) & 255] & 3;
    ring[w][i] = MODE >= 1 ? (uint32_t)(c0 | 0x80 | ((4 + c1) << 8) | 0x8000) : (uint32_t)c0;
  }
  __syncwarp();
  uint32_t tabA[P], tabB[P];   // MODE 1: byte k = [row p (P+p) has code k]
  uint32_t mpk = 0;            // MODE 0: byte k = rows with code k
  for (int p = 0; p < P; ++p) {
    tabA[p] = 0; tabB[p] = 0;
    for (int k = 0; k < 4; ++k) {
      tabA[p] |= (uint32_t)(code[p] == k) << (8 * k);
      tabB[p] |= (uint32_t)(code[P + p] == k) << (8 * k);
    }
  }
  for (int r = 0; r < R; ++r) mpk |= 1u << (8 * code[r] + r);
  const uint32_t one = (uint32_t)(n >> 30) | 1u;
  long long t0 = clock64();
  uint32_t acc = 0;
  if (MODE == 2) {
    uint32_t h[P];
    uint32_t fifo[E];
    for (int p = 0; p < P; ++p) h[p] = 0;
    for (int d = 0; d < E; ++d) fifo[d] = 0;
    uint32_t U0p = 0;
    const uint32_t inj = 0;
    const uint32_t ssel = lane == 31 ? 0x1054u : 0x3210u;   // lane 31: (inj lo, own A lo)
    for (int t = 0; t < n; t += 8) {
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t s = ring[w][((t - lane * EL) & 255) + u];
        const uint32_t U0 = fifo[E - 1];
        uint32_t U = U0, UL = U0p;
        uint32_t nw[P];
#pragma unroll
        for (int p = 0; p < P; ++p) {
          const uint32_t m = prmt(tabA[p], tabB[p], s);
          const uint32_t X = imad(m, one, UL);
          const uint32_t v = __vimax3_u16x2(U, h[p], X);
          UL = h[p];
          U = v;
          nw[p] = v;
        }
        U0p = U0;
        const uint32_t sv = prmt(nw[P - 1], inj, ssel);
        const uint32_t rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
        for (int d = E - 1; d > 0; --d) fifo[d] = fifo[d - 1];
        fifo[0] = rv;
#pragma unroll
        for (int p = 0; p < P; ++p) h[p] = nw[p];
      }
    }
    for (int p = 0; p < P; ++p) acc += h[p];
  } else if (MODE == 1) {
    uint32_t h[P];
    uint32_t fifo[E + 1];
    uint32_t U0p = 0, lol1 = 0;
    for (int p = 0; p < P; ++p) h[p] = 0;
    for (int d = 0; d <= E; ++d) fifo[d] = 0;
    const uint32_t inj = 0;
    for (int t = 0; t < n; t += 8) {
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t s = ring[w][((t - lane * EL) & 255) + u];
        // U of pair 0: lo = row 2P-1 of lane k-1 at column c (hi half of what it sent E steps ago),
        // hi = own row P-1 at column c-1 (lo half of the last pair one step ago)
        const uint32_t U0 = imadhi(fifo[E - 1], 0x10000u, lol1 << 16);
        uint32_t U = U0, UL = U0p;
        uint32_t nw[P];
#pragma unroll
        for (int p = 0; p < P; ++p) {
          const uint32_t m = prmt(tabA[p], tabB[p], s);
          const uint32_t X = imad(m, one, UL);
          const uint32_t v = __vimax3_u16x2(U, h[p], X);
          UL = h[p];
          U = v;
          nw[p] = v;
        }
        U0p = U0;
        lol1 = nw[P - 1];
        const uint32_t sv = (lane == 31) ? inj : nw[P - 1];
        const uint32_t rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
        for (int d = E; d > 0; --d) fifo[d] = fifo[d - 1];
        fifo[0] = rv;
#pragma unroll
        for (int p = 0; p < P; ++p) h[p] = nw[p];
      }
    }
    for (int p = 0; p < P; ++p) acc += h[p];
  } else {
    int h[R];
    int fifo[E + 1];
    for (int r = 0; r < R; ++r) h[r] = 0;
    for (int d = 0; d <= E; ++d) fifo[d] = 0;
    for (int t = 0; t < n; t += 8) {
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t cd = ring[w][((t - lane * EL) & 255) + u];
        const uint32_t mk = __byte_perm(mpk, 0u, cd);
        int U = fifo[E - 1], UL = fifo[E];
        int nw[R];
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int ulp = (int)imad((uint32_t)UL, one, one);
          const int X = ((mk >> r) & 1u) ? ulp : UL;
          const int v = max(max(U, h[r]), X);
          UL = h[r];
          U = v;
          nw[r] = v;
        }
        const int sv = (lane == 31) ? 0 : nw[R - 1];
        const int rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
        for (int d = E; d > 0; --d) fifo[d] = fifo[d - 1];
        fifo[0] = rv;
#pragma unroll
        for (int r = 0; r < R; ++r) h[r] = nw[r];
      }
    }
    for (int r = 0; r < R; ++r) acc += (uint32_t)h[r];
  }
  long long t1 = clock64();
  out[blockIdx.x * 128 + threadIdx.x] = acc;
  if (lane == 0) cyc[blockIdx.x * 4 + w] = t1 - t0;
}

template <int P, int E, int MODE>
void run(const uint8_t* b, const uint8_t* a, uint32_t* out, long long* cyc, int n) {
  for (int rep = 0; rep < 2; ++rep) sweep<P, E, MODE><<<148, 128>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[148 * 4];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148 * 4; ++i) s += (double)h[i];
  s /= 148 * 4;
  printf("MODE=%d rows=%d E=%d: %.1f cycles/step, %.2f cells/cycle/SMSP\n", MODE, 2 * P, E, s / n,
         32.0 * 2 * P / (s / n));
}

int main() {
  const int n = 1 << 16;
  uint8_t *b, *a;
  uint32_t* out;
  long long* cyc;
  cudaMalloc(&b, 256);
  cudaMalloc(&a, 148 * 128 * 16);
  cudaMalloc(&out, 148 * 128 * 4);
  cudaMalloc(&cyc, 148 * 4 * 8);
  uint8_t hb[256], ha[148 * 128 * 16];
  uint32_t x = 12345;
  for (auto& v : hb) { x = x * 1664525u + 1013904223u; v = "ACGT"[x >> 30]; }
  for (auto& v : ha) { x = x * 1664525u + 1013904223u; v = "ACGT"[x >> 30]; }
  cudaMemcpy(b, hb, 256, cudaMemcpyHostToDevice);
  cudaMemcpy(a, ha, sizeof(ha), cudaMemcpyHostToDevice);
  run<3, 2, 2>(b, a, out, cyc, n);
  run<3, 3, 2>(b, a, out, cyc, n);
  run<3, 4, 2>(b, a, out, cyc, n);
  run<4, 3, 2>(b, a, out, cyc, n);
  run<2, 2, 2>(b, a, out, cyc, n);
  run<3, 2, 0>(b, a, out, cyc, n);
  run<3, 3, 0>(b, a, out, cyc, n);
  run<3, 2, 1>(b, a, out, cyc, n);
  run<3, 3, 1>(b, a, out, cyc, n);
  run<3, 4, 1>(b, a, out, cyc, n);
  run<4, 2, 1>(b, a, out, cyc, n);
  run<4, 3, 1>(b, a, out, cyc, n);
  run<2, 3, 1>(b, a, out, cyc, n);
  run<2, 2, 1>(b, a, out, cyc, n);
  return 0;
}
