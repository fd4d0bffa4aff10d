// step3.cu -- where does a lane-systolic LCS step spend its cycles?  One warp per SM
// sub-partition (4 warps / CTA, one CTA per SM), each sweeping its own private strip (no
// links).  Development tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o step3 step3.cu && ./step3
// MODE 0: rotate SHFL + per-step injection SHFL (the adiag body)
// MODE 1: rotate SHFL only (lane 31 sends its own bottom row)
// MODE 2: no SHFL (U from the lane's own register: pure chain + issue)
// MODE 3: rotate SHFL; injection value for lane 31 from shared memory (LDS), no second SHFL
// MODE 4: as 1 with the cell as t = VIADDMNMX(UL, m, L) off the chain, v = VIMNMX(U, t) on it
// MODE 5: as 4 without SHFL
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int R, int E, int MODE>
__global__ void __launch_bounds__(256, 1) sweep(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a,
                                                int* out, long long* cyc) {

  __shared__ uint8_t sb[1 << 12];
  __shared__ int topv[8][1 << 8];
  __shared__ uint8_t mtab[8][64][32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < n && i < (1 << 12); i += blockDim.x) sb[i] = b[i];
  for (int i = threadIdx.x; i < 8 * (1 << 8); i += blockDim.x) (&topv[0][0])[i] = i & 7;
  for (int i = threadIdx.x; i < 8 * 64 * 32; i += blockDim.x) (&mtab[0][0][0])[i] = (uint8_t)(i * 37);
  __syncthreads();
  uint32_t am = 0;   // lane's row chars packed (R <= 4 rows per word ... use compare per row)
  int ar[R];
  for (int r = 0; r < R; ++r) ar[r] = a[(blockIdx.x * blockDim.x + threadIdx.x) * R + r];
  (void)am;
  int hist[R];
  int fifo[E + 1];
  for (int r = 0; r < R; ++r) hist[r] = 0;
  for (int d = 0; d <= E; ++d) fifo[d] = 0;
  const int one = n >> 30 | 1;
  const int tvreg = lane;
  long long t0 = clock64();
  for (int t = 0; t < n; t += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int tt = t + u;
      const int cc = (MODE == 8) ? (int)mtab[w][sb[(tt - lane * E) & ((1 << 12) - 1)] & 63][lane] : sb[(tt - lane * E) & ((1 << 12) - 1)];
      int U = (MODE == 2 || MODE == 5) ? hist[R - 1] : fifo[E - 1];
      int UL = (MODE == 2 || MODE == 5) ? hist[0] : fifo[E];
      int nw[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int L = hist[r];
        int v;
        if (MODE == 8) {
          // the adiag LCS cell: match bit from the per-step mask, predicated IMAD, VIMNMX3
          const int ulp = UL * one + one;
          const int t2 = ((cc >> r) & 1) ? ulp : UL;
          v = max(max(U, L), t2);
        } else if (MODE >= 4) {
          // off-chain: t = max(UL + m, L) (one VIADDMNMX); on-chain: v = max(U, t)
          const int m = (ar[r] == cc) ? one : 0;
          const int t2 = __viaddmax_s32(UL, m, L);
          v = max(U, t2);
        } else {
          const int d = (ar[r] == cc) ? UL + one : UL;
          v = max(max(U, L), d);
        }
        UL = hist[r];
        U = v;
        nw[r] = v;
      }
      if (MODE != 2 && MODE != 5) {
        int sv = nw[R - 1];
        if (MODE == 0) {
          const int inj = __shfl_sync(0xffffffffu, tvreg, (tt & 7) + 8);
          sv = (lane == 31) ? inj : sv;
        } else if (MODE == 3) {
          const int inj = topv[w][tt & 255];
          sv = (lane == 31) ? inj : sv;
        }
        const int rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
        for (int d = E; d > 0; --d) fifo[d] = fifo[d - 1];
        fifo[0] = rv;
      }
#pragma unroll
      for (int r = 0; r < R; ++r) hist[r] = nw[r];
    }
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += hist[r];
  for (int d = 0; d <= E; ++d) acc += fifo[d];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (lane == 0) cyc[blockIdx.x * 8 + w] = t1 - t0;
}

template <int R, int E, int MODE>
void run(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n, int nw = 4) {
  sweep<R, E, MODE><<<148, nw * 32>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  sweep<R, E, MODE><<<148, nw * 32>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[148 * 8];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148; ++i)
    for (int w = 0; w < nw; ++w) s += (double)h[i * 8 + w];
  s /= 148 * nw;
  printf("R=%d E=%d MODE=%d NW=%d: %.1f cycles/step, %.2f cycles/cell/warp, %.2f cells/cycle/SMSP\n", R, E, MODE, nw,
         s / n, s / n / R, (nw / 4.0) * 32 * R / (s / n));
}

// Pair interleave: steps u and u+1 emitted together, u+1 one row behind (independent chains
// interleaved for the in-order issue).  SH = 1: rotate SHFL (lane 31 sends its own bottom row).
template <int R, int E, int SH>
__global__ void __launch_bounds__(128, 1) sweep2(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a,
                                                 int* out, long long* cyc) {
  __shared__ uint8_t sb[1 << 12];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < n && i < (1 << 12); i += blockDim.x) sb[i] = b[i];
  __syncthreads();
  int ar[R];
  for (int r = 0; r < R; ++r) ar[r] = a[(blockIdx.x * 128 + threadIdx.x) * R + r];
  int hist[R];
  int fifo[E + 2];
  for (int r = 0; r < R; ++r) hist[r] = 0;
  for (int d = 0; d < E + 2; ++d) fifo[d] = 0;
  const int one = n >> 30 | 1;
  long long t0 = clock64();
  for (int t = 0; t < n; t += 8) {
#pragma unroll
    for (int u = 0; u < 8; u += 2) {
      const int tt = t + u;
      const int c0 = sb[(tt - lane * E) & ((1 << 12) - 1)];
      const int c1 = sb[(tt + 1 - lane * E) & ((1 << 12) - 1)];
      // step tt: U0 = fifo[E-1], UL0 = fifo[E]; step tt+1: U1 = fifo[E-2] (received one step later)
      int U0 = SH ? fifo[E - 1] : hist[R - 1], UL0 = SH ? fifo[E] : hist[0];
      int U1 = SH ? fifo[E - 2] : hist[R - 2], UL1 = SH ? fifo[E - 1] : hist[1];
      int n0[R], n1[R];
#pragma unroll
      for (int r = 0; r <= R; ++r) {
        if (r < R) {
          const int L = hist[r];
          const int d = (ar[r] == c0) ? UL0 + one : UL0;
          const int v = max(max(U0, L), d);
          UL0 = L; U0 = v; n0[r] = v;
        }
        if (r >= 1) {
          const int q = r - 1;
          const int L = n0[q];
          const int d = (ar[q] == c1) ? UL1 + one : UL1;
          const int v = max(max(U1, L), d);
          UL1 = L; U1 = v; n1[q] = v;
        }
      }
      if (SH) {
        const int r0 = __shfl_sync(0xffffffffu, n0[R - 1], (lane + 31) & 31);
        const int r1 = __shfl_sync(0xffffffffu, n1[R - 1], (lane + 31) & 31);
#pragma unroll
        for (int d = E + 1; d > 1; --d) fifo[d] = fifo[d - 2];
        fifo[1] = r0;
        fifo[0] = r1;
      }
#pragma unroll
      for (int r = 0; r < R; ++r) hist[r] = n1[r];
    }
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += hist[r];
  for (int d = 0; d < E + 2; ++d) acc += fifo[d];
  out[blockIdx.x * 128 + threadIdx.x] = acc;
  if (lane == 0) cyc[blockIdx.x * 4 + w] = t1 - t0;
}

template <int R, int E, int SH>
void run2(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n) {
  sweep2<R, E, SH><<<148, 128>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  sweep2<R, E, SH><<<148, 128>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[148 * 4];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148 * 4; ++i) s += (double)h[i];
  s /= 148 * 4;
  printf("PAIR R=%d E=%d SH=%d: %.1f cycles/step, %.2f cycles/cell\n", R, E, SH, s / n, s / n / R);
}


// Two independent strips per thread (chains A and B share nothing), interleaved per row: if the
// step is latency-bound this doubles the cells per cycle.
template <int R, int E>
__global__ void __launch_bounds__(128, 1) sweep_dual(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a,
                                                     int* out, long long* cyc) {
  __shared__ uint8_t sb[1 << 12];
  __shared__ uint8_t mtab[4][64][32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < n && i < (1 << 12); i += blockDim.x) sb[i] = b[i];
  for (int i = threadIdx.x; i < 4 * 64 * 32; i += blockDim.x) (&mtab[0][0][0])[i] = (uint8_t)(i * 37);
  __syncthreads();
  int hA[R], hB[R], fA[E + 1], fB[E + 1];
  for (int r = 0; r < R; ++r) { hA[r] = 0; hB[r] = r; }
  for (int d = 0; d <= E; ++d) { fA[d] = 0; fB[d] = d; }
  const int one = n >> 30 | 1;
  long long t0 = clock64();
  for (int t = 0; t < n; t += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int tt = t + u;
      const int ca = mtab[w][sb[(tt - lane * E) & 4095] & 63][lane];
      const int cb = mtab[w][sb[(tt + 977 - lane * E) & 4095] & 63][lane];
      int UA = fA[E - 1], ULA = fA[E], UB = fB[E - 1], ULB = fB[E];
      int nA[R], nB[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        {
          const int L = hA[r];
          const int t2 = ((ca >> r) & 1) ? ULA * one + one : ULA;
          const int v = max(max(UA, L), t2);
          ULA = L; UA = v; nA[r] = v;
        }
        {
          const int L = hB[r];
          const int t2 = ((cb >> r) & 1) ? ULB * one + one : ULB;
          const int v = max(max(UB, L), t2);
          ULB = L; UB = v; nB[r] = v;
        }
      }
      const int ra = __shfl_sync(0xffffffffu, nA[R - 1], (lane + 31) & 31);
      const int rb = __shfl_sync(0xffffffffu, nB[R - 1], (lane + 31) & 31);
#pragma unroll
      for (int d = E; d > 0; --d) { fA[d] = fA[d - 1]; fB[d] = fB[d - 1]; }
      fA[0] = ra; fB[0] = rb;
#pragma unroll
      for (int r = 0; r < R; ++r) { hA[r] = nA[r]; hB[r] = nB[r]; }
    }
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += hA[r] + hB[r];
  for (int d = 0; d <= E; ++d) acc += fA[d] + fB[d];
  out[blockIdx.x * 128 + threadIdx.x] = acc;
  if (lane == 0) cyc[blockIdx.x * 8 + w] = t1 - t0;
}

template <int R, int E>
void run_dual(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n) {
  sweep_dual<R, E><<<148, 128>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  sweep_dual<R, E><<<148, 128>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[148 * 8];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148; ++i)
    for (int w = 0; w < 4; ++w) s += (double)h[i * 8 + w];
  s /= 148 * 4;
  printf("DUAL R=%d E=%d: %.1f cycles/step (2 strips), %.2f cells/cycle/SMSP\n", R, E, s / n, 2.0 * 32 * R / (s / n));
}


// SPLIT: a lane's R rows as two sub-chains of R/2; the lower half runs one column behind the
// upper half (its U at column c-1 was produced by the upper half one step earlier), so the two
// chains of a step are independent: ILP 2 for one extra step of lane lag.
template <int R, int E>
__global__ void __launch_bounds__(128, 1) sweep_split(const uint8_t* __restrict__ b, int n, const uint8_t* __restrict__ a,
                                                      int* out, long long* cyc) {
  constexpr int H2 = R / 2;
  __shared__ uint8_t sb[1 << 12];
  __shared__ uint8_t mtab[4][64][32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < n && i < (1 << 12); i += blockDim.x) sb[i] = b[i];
  for (int i = threadIdx.x; i < 4 * 64 * 32; i += blockDim.x) (&mtab[0][0][0])[i] = (uint8_t)(i * 37);
  __syncthreads();
  int hist[R], fifo[E + 1];
  for (int r = 0; r < R; ++r) hist[r] = 0;
  for (int d = 0; d <= E; ++d) fifo[d] = 0;
  int mid = 0;      // upper half's last row at the previous step (U for the lower half)
  int midUL = 0;    // ... two steps back (UL for the lower half)
  int cprev = 0;    // previous step's match mask (the lower half's column)
  const int one = n >> 30 | 1;
  long long t0 = clock64();
  for (int t = 0; t < n; t += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int tt = t + u;
      const int cc = (int)mtab[w][sb[(tt - lane * (E + 1)) & 4095] & 63][lane];
      int UA = fifo[E - 1], ULA = fifo[E];
      int UB = mid, ULB = midUL;
      int nw[R];
#pragma unroll
      for (int r = 0; r < H2; ++r) {
        {   // upper half, column c
          const int L = hist[r];
          const int t2 = ((cc >> r) & 1) ? ULA * one + one : ULA;
          const int v = max(max(UA, L), t2);
          ULA = L; UA = v; nw[r] = v;
        }
        {   // lower half, column c - 1
          const int q = H2 + r;
          const int L = hist[q];
          const int t2 = ((cprev >> q) & 1) ? ULB * one + one : ULB;
          const int v = max(max(UB, L), t2);
          ULB = L; UB = v; nw[q] = v;
        }
      }
      midUL = hist[H2 - 1];
      mid = nw[H2 - 1];
      cprev = cc;
      const int rv = __shfl_sync(0xffffffffu, nw[R - 1], (lane + 31) & 31);
#pragma unroll
      for (int d = E; d > 0; --d) fifo[d] = fifo[d - 1];
      fifo[0] = rv;
#pragma unroll
      for (int r = 0; r < R; ++r) hist[r] = nw[r];
    }
  }
  long long t1 = clock64();
  int acc = 0;
  for (int r = 0; r < R; ++r) acc += hist[r];
  for (int d = 0; d <= E; ++d) acc += fifo[d];
  out[blockIdx.x * 128 + threadIdx.x] = acc;
  if (lane == 0) cyc[blockIdx.x * 8 + w] = t1 - t0;
}

template <int R, int E>
void run_split(const uint8_t* b, const uint8_t* a, int* out, long long* cyc, int n) {
  sweep_split<R, E><<<148, 128>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  sweep_split<R, E><<<148, 128>>>(b, n, a, out, cyc);
  cudaDeviceSynchronize();
  long long h[148 * 8];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < 148; ++i)
    for (int w = 0; w < 4; ++w) s += (double)h[i * 8 + w];
  s /= 148 * 4;
  printf("SPLIT R=%d E=%d: %.1f cycles/step, %.2f cycles/cell\n", R, E, s / n, s / n / R);
}

int main() {
  const int n = 1 << 14;
  uint8_t *b, *a;
  int* out;
  long long* cyc;
  cudaMalloc(&b, 1 << 16);
  cudaMalloc(&a, 148 * 256 * 16);
  cudaMalloc(&out, 148 * 256 * 4);
  cudaMalloc(&cyc, 148 * 8 * 8);
  cudaMemset(b, 1, 1 << 16);
  cudaMemset(a, 1, 148 * 256 * 16);
  run_split<6, 2>(b, a, out, cyc, n);
  run_split<8, 2>(b, a, out, cyc, n);
  run_split<12, 2>(b, a, out, cyc, n);
  run_split<6, 1>(b, a, out, cyc, n);
  run_dual<6, 2>(b, a, out, cyc, n);
  run_dual<4, 2>(b, a, out, cyc, n);
  run_dual<3, 2>(b, a, out, cyc, n);
  run_dual<8, 2>(b, a, out, cyc, n);
  run<6, 2, 0>(b, a, out, cyc, n);
  run<6, 2, 8>(b, a, out, cyc, n);
  run<6, 2, 2>(b, a, out, cyc, n);
  run<6, 2, 8>(b, a, out, cyc, n, 8);
  run<3, 2, 8>(b, a, out, cyc, n, 8);
  run<4, 2, 8>(b, a, out, cyc, n, 8);
  run<6, 2, 2>(b, a, out, cyc, n, 8);
  run<4, 2, 8>(b, a, out, cyc, n);
  run<8, 2, 8>(b, a, out, cyc, n);
  run<12, 3, 8>(b, a, out, cyc, n);
  run<16, 3, 8>(b, a, out, cyc, n);
  run2<6, 2, 1>(b, a, out, cyc, n);
  return 0;
}
