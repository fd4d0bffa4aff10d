// prevrow.cuh -- previous-row-only ("Horizontal", t = i) category kernel [L180-L195], Fig. 2(b).
//
// Every cell of row i depends only on row i-1 (contributing set within {UL, U, UR}); the
// degree of parallelism is the row width in every iteration [L184].  The paper runs one
// launch per row [L184], [L251].  Here ONE persistent launch fills the whole table:
//
//  * TASKS = (band b, column block J): rows [b*h, (b+1)*h) x columns [J*BW, (J+1)*BW).  A warp
//    claims tasks in increasing band-major order (atomic counter), so every task waits only on
//    tasks claimed earlier -- deadlock-free without co-residency -- and the bands pipeline.
//  * A task computes the TRAPEZOID of its block: it starts from row b*h-1 over the extended
//    window [J*BW - h, (J+1)*BW + h) (read from the previous band's boundary row, L2) and
//    recomputes the h-column halo on each side, which is garbage-free for the block's own
//    columns after h rows.  This is the case-2 two-way halo of Table II [L265-L274]
//    ([L193-L195]): no per-row exchange between blocks at all.
//  * Inside the warp each lane owns VP = BW/32 + 2h/32 consecutive columns; UL / UR across
//    lanes come from __shfl_up / __shfl_down every row.  Cost rows are streamed with a
//    software-pipelined register prefetch ring (rows r+1..r+PF in flight).
//  * Boundary rows go to a 4-deep ring of global rows with an epoch-tagged release flag per
//    block (its completed band count).
#pragma once
#include <cstdint>
#include <climits>
#include "cellfn.cuh"
#include "params.h"
#include "sync.cuh"

namespace lddp {

constexpr int kPrevBandRows = 64;   // h  (band rows = halo columns)
constexpr int kPrevV = 4;           // own columns per lane: BW = 128
constexpr int kPrevWarps = 8;
constexpr int kPrevRing = 4;        // boundary-row ring depth
constexpr int kPrevPF = 4;          // cost-row prefetch distance

template <class F, bool TABLE>
__global__ void __launch_bounds__(kPrevWarps * 32) prevrow_kernel(const FillParams p) {
  using T = typename F::T;
  using G = typename F::GridT;
  constexpr int h = kPrevBandRows;
  constexpr int VP = kPrevV + 2 * h / 32;  // columns per lane in the extended window
  constexpr int BW = 32 * kPrevV;
  static_assert(!(F::kMask & NB_L), "prev-row category: f must not read L");

  Control* ctl = static_cast<Control*>(p.ctl);
  const uint64_t tmo = p.timeout_ns;
  const int lane = threadIdx.x & 31;
  const int W = p.cols;
  const int64_t H = p.rows;
  const int nb = p.nblocks;
  const int nbands = p.nstrips;
  const uint64_t ep = p.epoch << 32;
  const int64_t ntasks = (int64_t)nb * nbands;
  T* ring = static_cast<T*>(p.bnd);
  unsigned* rowmin_done = &ctl->pad[0];
  T* rowmins = reinterpret_cast<T*>(p.prog + nb);   // nb entries after the flags

  while (true) {
    int64_t t = 0;
    if (lane == 0) t = (int64_t)atomicAdd(&ctl->claim, 1u);
    t = __shfl_sync(0xffffffffu, t, 0);
    if (t >= ntasks) break;
    const int b = (int)(t / nb);
    const int J = (int)(t % nb);
    const int j0 = J * BW;
    const int e0 = j0 - h + lane * VP;     // first column of this lane
    const int64_t r0 = (int64_t)b * h;     // first row of the band

    // ---- input row r0 - 1 over the extended window
    T cur[VP];
    if (b == 0) {
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        const int col = e0 + v;
        cur[v] = (col < 0) ? F::left(p, -1) : (col >= W ? F::right(p, -1) : F::top(p, col));
      }
    } else {
      const uint64_t need = ep | (uint64_t)b;
      bool ok = true;
      if (J > 0) ok = ok && wait_flag<false>(p.prog + (J - 1), need, ctl, tmo);
      ok = ok && wait_flag<false>(p.prog + J, need, ctl, tmo);
      if (J + 1 < nb) ok = ok && wait_flag<false>(p.prog + (J + 1), need, ctl, tmo);
      if (!ok) return;
      const T* src = ring + (int64_t)((b - 1) % kPrevRing) * p.bnd_stride;
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        const int col = e0 + v;
        cur[v] = (col < 0) ? F::left(p, r0 - 1) : (col >= W ? F::right(p, r0 - 1) : __ldcg(src + col));
      }
    }

    // ---- prefetch ring of cost rows
    G pf[kPrevPF][VP];
#pragma unroll
    for (int d = 0; d < kPrevPF; ++d) {
      const int64_t row = r0 + d;
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        const int col = e0 + v;
        pf[d][v] = (row < H && col >= 0 && col < W) ? F::load(p, row, col) : G(0);
      }
    }

    const int nrows = (int)((r0 + h <= H) ? h : (H - r0));
#pragma unroll
    for (int r = 0; r < h; ++r) {
      if (r >= nrows) break;
      const int64_t row = r0 + r;
      G g[VP];
#pragma unroll
      for (int v = 0; v < VP; ++v) g[v] = pf[r % kPrevPF][v];
      {
        const int64_t prow = row + kPrevPF;
#pragma unroll
        for (int v = 0; v < VP; ++v) {
          const int col = e0 + v;
          pf[r % kPrevPF][v] = (prow < r0 + nrows && col >= 0 && col < W) ? F::load(p, prow, col) : G(0);
        }
      }
      const T lv = __shfl_up_sync(0xffffffffu, cur[VP - 1], 1);
      const T rv = __shfl_down_sync(0xffffffffu, cur[0], 1);
      T nw[VP];
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        const int col = e0 + v;
        const T UL = (v > 0) ? cur[v - 1] : lv;
        const T U = cur[v];
        const T UR = (v < VP - 1) ? cur[v + 1] : rv;
        typename F::OutT o;
        T x = F::f(U, UL, U, UR, typename F::RowCtx(0), typename F::ColCtx(0), g[v], row, col,
                   p.param_c, o);
        if (col < 0) x = F::left(p, row);
        if (col >= W) x = F::right(p, row);
        if (TABLE && col >= j0 && col < j0 + BW && col < W)
          static_cast<typename F::OutT*>(p.table)[row * p.table_pitch + col] = o;
        nw[v] = x;
      }
#pragma unroll
      for (int v = 0; v < VP; ++v) cur[v] = nw[v];
    }

    // ---- publish the block's bottom row (or the outputs for the last band)
    const bool last_band = (b == nbands - 1);
    if (!last_band) {
      T* dst = ring + (int64_t)(b % kPrevRing) * p.bnd_stride;
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        const int col = e0 + v;
        if (col >= j0 && col < j0 + BW && col < W) __stcg(dst + col, cur[v]);
      }
      __threadfence();
      __syncwarp();
      if (lane == 0) st_release_gpu(p.prog + J, ep | (uint64_t)(b + 1));
    } else {
      T mn = INT_MAX;
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        const int col = e0 + v;
        if (col >= j0 && col < j0 + BW && col < W) {
          if (p.last_row != nullptr) static_cast<T*>(p.last_row)[col] = cur[v];
          mn = min(mn, cur[v]);
        }
      }
      if (F::kScore == SCORE_ROW_MIN && p.score != nullptr) {
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, off));
        if (lane == 0) {
          rowmins[J] = mn;
          __threadfence();
          const unsigned d = atomicAdd(rowmin_done, 1u);
          if (d == (unsigned)nb - 1) {
            __threadfence();
            T best = INT_MAX;
            for (int k = 0; k < nb; ++k) best = min(best, __ldcg(rowmins + k));
            *static_cast<T*>(p.score) = best;
            atomicExch(rowmin_done, 0u);
          }
        }
      }
    }
  }
  // last warp out resets the claim counter for the next fill
  if (lane == 0) {
    __threadfence();
    const unsigned total = gridDim.x * (blockDim.x / 32);
    const unsigned d = atomicAdd(&ctl->done, 1u);
    if (d == total - 1) {
      atomicExch(&ctl->claim, 0u);
      atomicExch(&ctl->done, 0u);
    }
  }
}

}  // namespace lddp
