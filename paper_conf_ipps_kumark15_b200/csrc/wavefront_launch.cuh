// wavefront_launch.cuh -- instantiation / dispatch helpers for wavefront_kernel.
//
// Geometry variants (rows per lane R, intra-lane skew SIG, extra lane lag E, compute warps W).
// The planner picks one; every variant is bit-identical (same cells, same per-cell arithmetic).
#pragma once
#include "wavefront.cuh"

namespace lddp {

enum WfVariant : int {
  WF_A_R4_S0 = 0,   // anti-diagonal: 4 rows / lane, rows chained within a step, E = 2
  WF_A_R4_S1 = 1,   // anti-diagonal: 4 rows / lane, rows skewed one step, E = 1
  WF_A_R2_S1 = 2,   // anti-diagonal: 2 rows / lane, skewed
  WF_A_R8_S1 = 3,   // anti-diagonal: 8 rows / lane, skewed
  WF_A_R8_S0 = 4,   // anti-diagonal: 8 rows / lane, chained, E = 2
  WF_A_R4_E1 = 5,   // anti-diagonal: 4 rows / lane, chained, E = 1
  WF_A_R16_S0 = 6,  // anti-diagonal: 16 rows / lane, chained, E = 2
  WF_A_R8_E3 = 7,   // anti-diagonal: 8 rows / lane, chained, E = 3
  WF_A_R8_G4 = 8,   // anti-diagonal: 8 rows / lane = 2 chained groups of 4, groups skewed 1, E = 1
  WF_A_R8_G2 = 9,   // anti-diagonal: 8 rows / lane = 4 chained groups of 2, skewed 1, E = 1
  WF_A_R16_G4 = 12, // anti-diagonal: 16 rows / lane = 4 chained groups of 4, skewed 1, E = 1
  WF_K_R1 = 10,     // knight-move: 1 row / lane, skew 2, E = 2
  WF_K_R2 = 11,     // knight-move: 2 rows / lane, skew 2, E = 2
  WF_K_R1_E1 = 13,  // knight-move: 1 row / lane, skew 2, E = 1 (D = 3)
};
constexpr int kWfWarps = 4;

template <class F, int R, int SIG, int E, int W, bool TABLE, int GS>
inline cudaError_t wf_launch(const FillParams& p, int grid, cudaStream_t s) {
  wavefront_kernel<F, R, SIG, E, W, TABLE, GS><<<grid, Wave<F, R, SIG, E, W, TABLE, GS>::kThreads, 0, s>>>(p);
  return cudaGetLastError();
}

template <class F, int R, int SIG, int E, int W, bool TABLE, int GS>
inline int wf_occ() {
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(
          &n, wavefront_kernel<F, R, SIG, E, W, TABLE, GS>, Wave<F, R, SIG, E, W, TABLE, GS>::kThreads, 0) !=
      cudaSuccess)
    return 0;
  return n;
}

// Per-function dispatchers (one translation unit each).  op = 0: launch, 1: occupancy query,
// 2: "is this (variant, table) compiled?".
#define LDDP_WF_DECL(name)                                                                     \
  int wf_dispatch_##name(int op, int variant, bool table, const FillParams* p, int grid,       \
                         cudaStream_t s)
LDDP_WF_DECL(lcs);
LDDP_WF_DECL(lev);
LDDP_WF_DECL(dtw);
LDDP_WF_DECL(fs);
LDDP_WF_DECL(minpath3);
LDDP_WF_DECL(min2plus);
LDDP_WF_DECL(diagmaxplus);

#define LDDP_WF_CASE_G(F, V, R, SIG, E, TABLE, G)                                              \
  if (variant == (V) && table == (TABLE)) {                                                    \
    if (op == 0) return (int)wf_launch<F, R, SIG, E, kWfWarps, TABLE, G>(*p, grid, s);         \
    if (op == 1) return wf_occ<F, R, SIG, E, kWfWarps, TABLE, G>();                            \
    return 1;                                                                                  \
  }
#define LDDP_WF_CASE(F, V, R, SIG, E, TABLE) LDDP_WF_CASE_G(F, V, R, SIG, E, TABLE, ((SIG) == 0 ? (R) : 1))

}  // namespace lddp
