// traceback.cu -- traceback of an anti-diagonal fill's TABLE output (LCS, Levenshtein, DTW):
// SURVEY §8(f) NEXT #2.  One thread walks from DP cell (m, n) back towards the boundary, reading
// the f-evaluated region T[i-1][j-1] = D[i][j] (row / column 0 implied by f's initialisation,
// DESIGN.md R-TB).  O(m + n) dependent steps: an output mode for moderate sizes, not the hot path.
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

__global__ void traceback_kernel(int func, const void* a, const void* b, const void* table, int64_t pitch, int64_t m,
                                 int64_t n, int32_t* pi, int32_t* pj, int64_t* len) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  int64_t i = m, j = n, k = 0;
  if (func == 1) {   // DTW
    const float* t = static_cast<const float*>(table);
    const float inf = INFINITY;
    while (i >= 1 && j >= 1) {
      pi[k] = (int32_t)i;
      pj[k] = (int32_t)j;
      ++k;
      if (i == 1 && j == 1) break;
      const float d = tb_at<float>(t, pitch, i - 1, j - 1, 0.0f, inf, inf, 2);
      const float u = tb_at<float>(t, pitch, i - 1, j, 0.0f, inf, inf, 2);
      const float l = tb_at<float>(t, pitch, i, j - 1, 0.0f, inf, inf, 2);
      if (d <= u && d <= l) { --i; --j; }
      else if (u <= l) { --i; }
      else { --j; }
    }
  } else {
    const int32_t* t = static_cast<const int32_t*>(table);
    const uint8_t* sa = static_cast<const uint8_t*>(a);
    const uint8_t* sb = static_cast<const uint8_t*>(b);
    const int kind = (func == 6) ? 1 : 0;   // LDDP_F_LEVENSHTEIN = 6, LCS = 0
    while (i >= 1 && j >= 1) {
      pi[k] = (int32_t)i;
      pj[k] = (int32_t)j;
      ++k;
      const bool eq = sa[i - 1] == sb[j - 1];
      const int32_t dd = tb_at<int32_t>(t, pitch, i - 1, j - 1, 0, 0, 0, kind);
      const int32_t du = tb_at<int32_t>(t, pitch, i - 1, j, 0, 0, 0, kind);
      const int32_t dl = tb_at<int32_t>(t, pitch, i, j - 1, 0, 0, 0, kind);
      if (kind == 0) {
        if (eq) { --i; --j; }
        else if (du >= dl) { --i; }
        else { --j; }
      } else {
        const int32_t here = tb_at<int32_t>(t, pitch, i, j, 0, 0, 0, kind);
        if (eq && here == dd) { --i; --j; }
        else if (here == dd + 1) { --i; --j; }
        else if (here == du + 1) { --i; }
        else { --j; }
      }
    }
  }
  *len = k;
}

cudaError_t launch_traceback(int func, const void* a, const void* b, const void* table, int64_t pitch, int64_t m,
                             int64_t n, int32_t* pi, int32_t* pj, int64_t* len, cudaStream_t s) {
  traceback_kernel<<<1, 32, 0, s>>>(func, a, b, table, pitch, m, n, pi, pj, len);
  return cudaGetLastError();
}

}  // namespace lddp
