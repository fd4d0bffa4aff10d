// traceback.cu -- traceback of an anti-diagonal fill's TABLE output (LCS, Levenshtein, DTW):
// SURVEY §8(f) NEXT #2.  One thread walks from DP cell (m, n) back towards the boundary, reading
// the f-evaluated region T[i-1][j-1] = D[i][j] (row / column 0 implied by f's initialisation,
// DESIGN.md R-TB).  O(m + n) dependent steps, walked block by block (below).
//
// Rules (reading R14), path = the DP cells (i, j), 1 <= i <= m, 1 <= j <= n, visited:
//  * LCS (textbook, CLRS PRINT-LCS): a_i == b_j -> (i-1, j-1); else up if D[i-1][j] >= D[i][j-1],
//    else left; stop when i == 0 or j == 0.
//  * Levenshtein: diagonal if a_i == b_j and D[i][j] == D[i-1][j-1]; else the first of
//    substitution (D[i-1][j-1] + 1), deletion (D[i-1][j] + 1), insertion (D[i][j-1] + 1) equal to
//    D[i][j]; stop when i == 0 or j == 0 (the rest are pure deletions / insertions).
//  * DTW: stop after (1, 1); else the argmin of D[i-1][j-1], D[i-1][j], D[i][j-1] (ties in that
//    order; out-of-table neighbours are +inf).
#include <cstdint>
#include <cmath>
#include "params.h"

namespace lddp {

namespace {
template <class T>
__device__ __forceinline__ T tb_at(const T* t, int64_t pitch, int64_t i, int64_t j, T b0, T brow, T bcol, int kind) {
  // D[i][j] with DP indices; boundary per f
  if (i >= 1 && j >= 1) return __ldcg(t + (i - 1) * pitch + (j - 1));
  if (kind == 1) return (T)(i > j ? i : j);   // Levenshtein: D[i][0] = i, D[0][j] = j
  if (i == 0 && j == 0) return b0;
  return (i == 0) ? brow : bcol;
}
}  // namespace

// One warp.  The walk only ever moves up / left / up-left, so it runs block by block: the warp
// loads the (B+1) x (B+1) DP cells [i-B, i] x [j-B, j] around the current cell (33 coalesced row
// segments, all loads in flight at once) and the matching string characters into shared memory,
// then lane 0 walks inside the block until the path leaves it (>= B steps unless it reaches the
// boundary).  One HBM round trip per block instead of one per path step.
constexpr int kTbB = 32;

template <class T>
__device__ __forceinline__ T tb_cell(const T* t, int64_t pitch, int64_t i, int64_t j, T b0, T brow, T bcol, int kind) {
  // predicated load (no branch): every load of a block is in flight at once
  const bool in = i >= 1 && j >= 1;
  const T v = __ldcg(t + (in ? (i - 1) * pitch + (j - 1) : 0));
  T bd;
  if (kind == 1) bd = (T)(i > j ? i : j);   // Levenshtein: D[i][0] = i, D[0][j] = j
  else bd = (i == 0 && j == 0) ? b0 : ((i == 0) ? brow : bcol);
  return in ? v : bd;
}

template <class T>
__device__ __forceinline__ void tb_load_block(const T* t, int64_t pitch, int64_t i0, int64_t j0, T b0, T brow, T bcol,
                                              int kind, const uint8_t* sa, const uint8_t* sb, T (*tile)[kTbB + 2],
                                              uint8_t* sas, uint8_t* sbs, int lane) {
  // lane c loads column j0 + c of the 33 rows (one coalesced segment per row, all in flight),
  // then lane r loads row i0 + r of column j0 + 32; cells outside the DP table are never read
  T v[kTbB + 1];
#pragma unroll
  for (int r = 0; r <= kTbB; ++r) v[r] = tb_cell<T>(t, pitch, i0 + r, j0 + lane, b0, brow, bcol, kind);
  const T e = tb_cell<T>(t, pitch, i0 + lane, j0 + kTbB, b0, brow, bcol, kind);
  const T e2 = tb_cell<T>(t, pitch, i0 + kTbB, j0 + kTbB, b0, brow, bcol, kind);
#pragma unroll
  for (int r = 0; r <= kTbB; ++r) tile[r][lane] = v[r];
  tile[lane][kTbB] = e;
  if (lane == 0) tile[kTbB][kTbB] = e2;
  if (sa != nullptr) {
    const int64_t ia = i0 + lane, jb = j0 + lane;
    sas[lane] = sa[ia >= 1 ? ia - 1 : 0];
    sbs[lane] = sb[jb >= 1 ? jb - 1 : 0];
    if (lane == 0) {
      sas[kTbB] = sa[i0 + kTbB >= 1 ? i0 + kTbB - 1 : 0];
      sbs[kTbB] = sb[j0 + kTbB >= 1 ? j0 + kTbB - 1 : 0];
    }
  }
  __syncwarp();
}

__global__ void traceback_kernel(int func, const void* a, const void* b, const void* table, int64_t pitch, int64_t m,
                                 int64_t n, int32_t* pi, int32_t* pj, int64_t* len) {
  if (blockIdx.x != 0) return;
  const int lane = threadIdx.x & 31;
  __shared__ union {
    float f[kTbB + 1][kTbB + 2];
    int32_t s[kTbB + 1][kTbB + 2];
  } tile;
  __shared__ uint8_t sas[kTbB + 1], sbs[kTbB + 1];
  int64_t i = m, j = n, k = 0;
  bool done = false;
  if (func == 1) {   // DTW
    const float* t = static_cast<const float*>(table);
    const float inf = INFINITY;
    while (!done && i >= 1 && j >= 1) {
      const int64_t i0 = i - kTbB, j0 = j - kTbB;
      tb_load_block<float>(t, pitch, i0, j0, 0.0f, inf, inf, 2, nullptr, nullptr, tile.f, sas, sbs, lane);
      if (lane == 0) {
        while (i > i0 && j > j0 && i >= 1 && j >= 1) {
          pi[k] = (int32_t)i;
          pj[k] = (int32_t)j;
          ++k;
          if (i == 1 && j == 1) { done = true; break; }
          const int ri = (int)(i - i0), cj = (int)(j - j0);
          const float d = tile.f[ri - 1][cj - 1], u = tile.f[ri - 1][cj], l = tile.f[ri][cj - 1];
          if (d <= u && d <= l) { --i; --j; }
          else if (u <= l) { --i; }
          else { --j; }
        }
      }
      i = __shfl_sync(0xffffffffu, i, 0);
      j = __shfl_sync(0xffffffffu, j, 0);
      k = __shfl_sync(0xffffffffu, k, 0);
      done = __shfl_sync(0xffffffffu, done, 0);
      __syncwarp();
    }
  } else {
    const int32_t* t = static_cast<const int32_t*>(table);
    const uint8_t* sa = static_cast<const uint8_t*>(a);
    const uint8_t* sb = static_cast<const uint8_t*>(b);
    const int kind = (func == 6) ? 1 : 0;   // LDDP_F_LEVENSHTEIN = 6, LCS = 0
    while (i >= 1 && j >= 1) {
      const int64_t i0 = i - kTbB, j0 = j - kTbB;
      tb_load_block<int32_t>(t, pitch, i0, j0, 0, 0, 0, kind, sa, sb, tile.s, sas, sbs, lane);
      if (lane == 0) {
        while (i > i0 && j > j0 && i >= 1 && j >= 1) {
          pi[k] = (int32_t)i;
          pj[k] = (int32_t)j;
          ++k;
          const int ri = (int)(i - i0), cj = (int)(j - j0);
          const bool eq = sas[ri] == sbs[cj];
          const int32_t dd = tile.s[ri - 1][cj - 1], du = tile.s[ri - 1][cj], dl = tile.s[ri][cj - 1];
          if (kind == 0) {
            if (eq) { --i; --j; }
            else if (du >= dl) { --i; }
            else { --j; }
          } else {
            const int32_t here = tile.s[ri][cj];
            if (eq && here == dd) { --i; --j; }
            else if (here == dd + 1) { --i; --j; }
            else if (here == du + 1) { --i; }
            else { --j; }
          }
        }
      }
      i = __shfl_sync(0xffffffffu, i, 0);
      j = __shfl_sync(0xffffffffu, j, 0);
      k = __shfl_sync(0xffffffffu, k, 0);
      __syncwarp();
    }
  }
  if (lane == 0) *len = k;
}

cudaError_t launch_traceback(int func, const void* a, const void* b, const void* table, int64_t pitch, int64_t m,
                             int64_t n, int32_t* pi, int32_t* pj, int64_t* len, cudaStream_t s) {
  traceback_kernel<<<1, 32, 0, s>>>(func, a, b, table, pitch, m, n, pi, pj, len);
  return cudaGetLastError();
}

}  // namespace lddp
