// prevrow.cu -- the previous-row-only kernels' TMA variant and the per-f launchers; the generic
// claimed-task kernel lives in prevrow.cuh (also instantiated by include/lddp_user.cuh).
#include "prevrow.cuh"

namespace lddp {

// ---------------------------------------------------------------------------------------------
// TMA variant (the default when W % 4 == 0 and the grid rows are 16-byte aligned): each warp
// streams its tasks' cost rows (the extended window, 768 B per row) into a 16-row shared-memory
// ring with cp.async.bulk + mbarrier complete_tx, issued up to 16 rows ahead of the row being
// computed and across task boundaries (the next task is claimed early), so HBM latency is hidden
// by the copy engine instead of by register prefetch.  The cell arithmetic is the same as above.
constexpr int kPrTmaWarps = 4;
constexpr int kPrRing = 16;

template <class F, bool TABLE>
__global__ void __launch_bounds__(kPrTmaWarps * 32) prevrow_tma_kernel(const FillParams p) {
  using T = typename F::T;
  using G = typename F::GridT;
  constexpr int h = kPrevBandRows;
  constexpr int VP = kPrevV + 2 * h / 32;
  constexpr int BW = 32 * kPrevV;
  constexpr int EXT = 32 * VP;
  static_assert(sizeof(G) == 4, "TMA prev-row path streams 32-bit costs");
  extern __shared__ __align__(128) unsigned char pr_smem[];
  using RingT = G[kPrRing][EXT];
  RingT* ring = reinterpret_cast<RingT*>(pr_smem);                                   // [warps]

  Control* ctl = static_cast<Control*>(p.ctl);
  const uint64_t tmo = p.timeout_ns;
  const int lane = threadIdx.x & 31;
  const int wl = threadIdx.x >> 5;
  const int W = p.cols;
  const int64_t H = p.rows;
  const int nb = p.nblocks;
  const int nbands = p.nstrips;
  const uint64_t ep = p.epoch << 32;
  const int64_t ntasks = (int64_t)nb * nbands;
  T* bring = static_cast<T*>(p.bnd);
  unsigned* rowmin_done = &ctl->pad[0];
  T* rowmins = reinterpret_cast<T*>(p.prog + nb);
  const G* cost = static_cast<const G*>(p.grid);


  auto claim = [&]() -> int64_t {
    int64_t t = 0;
    if (lane == 0) t = (int64_t)atomicAdd(&ctl->claim, 1u);
    return __shfl_sync(0xffffffffu, t, 0);
  };
  auto task_rows = [&](int64_t t) -> int {
    const int64_t r0 = (t / nb) * (int64_t)h;
    return (int)((r0 + h <= H) ? h : (H - r0));
  };

  // Claimed tasks: t_cur (being computed) and t_nxt (claimed by the issue cursor when it runs
  // past the end of t_cur).  The issue cursor never runs beyond t_nxt.  Exactly one row is
  // issued (one cp.async group committed, possibly empty) per row consumed, kPrRing-1 ahead.
  int64_t t_cur = claim();
  if (t_cur < ntasks) {
    int64_t t_nxt = -1;
    int iss = 0;          // 0: issuing rows of t_cur, 1: of t_nxt
    bool iss_done = false;
    int ir = 0, i_rows = 0;
    uint32_t islot = 0, cslot = 0;
    const G* isrc[VP / 2];
    bool iin[VP / 2];
    auto set_issue_task = [&](int64_t it) {
      if (it >= ntasks) return;
      const int bb = (int)(it / nb), JJ = (int)(it - (int64_t)bb * nb);
      const int64_t row0 = (int64_t)bb * h;
      i_rows = (int)((row0 + h <= H) ? h : (H - row0));
      const int col = JJ * BW - h + lane * VP;
#pragma unroll
      for (int j = 0; j < VP / 2; ++j) {
        iin[j] = (col + 2 * j >= 0) && (col + 2 * j < W);
        isrc[j] = cost + row0 * p.grid_pitch + (iin[j] ? col + 2 * j : 0);
      }
    };
    set_issue_task(t_cur);
    auto issue_one = [&]() {
      const int64_t it = iss ? t_nxt : t_cur;
      if (it < ntasks && !iss_done) {
        G* dst = &ring[wl][islot % kPrRing][lane * VP];
#pragma unroll
        for (int j = 0; j < VP / 2; ++j) {
          cp_async_8(dst + 2 * j, isrc[j], iin[j] ? 8u : 0u);
          isrc[j] += p.grid_pitch;
        }
        ++islot;
        if (++ir == i_rows) {
          ir = 0;
          if (iss == 0) {
            iss = 1;
            t_nxt = claim();
            set_issue_task(t_nxt);
          } else {
            iss_done = true;
          }
        }
      }
      cp_async_commit();
    };
    for (int k = 0; k < kPrRing - 1; ++k) issue_one();
    while (t_cur < ntasks) {
      const int b = (int)(t_cur / nb);
      const int J = (int)(t_cur % nb);
      const int j0 = J * BW;
      const int e0 = j0 - h + lane * VP;
      const int64_t r0 = (int64_t)b * h;
      bool outside[VP];
      T outv[VP];
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        const int col = e0 + v;
        outside[v] = col < 0 || col >= W;
        outv[v] = col < 0 ? F::left(p, 0) : F::right(p, 0);
      }
      T cur[VP];
      if (b == 0) {
#pragma unroll
        for (int v = 0; v < VP; ++v) cur[v] = outside[v] ? outv[v] : F::top(p, e0 + v);
      } else {
        const uint64_t need = ep | (uint64_t)b;
        bool ok = true;
        uint64_t seen;
        if (J > 0) ok = ok && wait_flag_relaxed(p.prog + (J - 1), need, ctl, tmo, seen);
        ok = ok && wait_flag_relaxed(p.prog + J, need, ctl, tmo, seen);
        if (J + 1 < nb) ok = ok && wait_flag_relaxed(p.prog + (J + 1), need, ctl, tmo, seen);
        if (!ok) return;
        const T* src = bring + (int64_t)((b - 1) % kPrevRing) * p.bnd_stride;
#pragma unroll
        for (int v = 0; v < VP; ++v) cur[v] = outside[v] ? outv[v] : __ldcg(src + e0 + v);
      }
      if (lane == 0 && p.trace != nullptr && J < p.trace_chunks)
        p.trace[((int64_t)b * p.trace_chunks + J) * 2] = globaltimer_ns();
      const int nrows = task_rows(t_cur);
      for (int r = 0; r < nrows; ++r) {
        issue_one();                           // row kPrRing-1 ahead (into the slot read last)
        cp_async_wait_group<kPrRing - 1>();    // this row's group has landed
        const int slot = cslot % kPrRing;
        const int64_t row = r0 + r;
        G g[VP];
#pragma unroll
        for (int v = 0; v < VP; ++v) g[v] = ring[wl][slot][lane * VP + v];
        ++cslot;
        const T lv = __shfl_up_sync(0xffffffffu, cur[VP - 1], 1);
        const T rv = __shfl_down_sync(0xffffffffu, cur[0], 1);
        T nw[VP];
#pragma unroll
        for (int v = 0; v < VP; ++v) {
          const T UL = (v > 0) ? cur[v - 1] : lv;
          const T U = cur[v];
          const T UR = (v < VP - 1) ? cur[v + 1] : rv;
          typename F::OutT o;
          T x = F::f(U, UL, U, UR, typename F::RowCtx(0), typename F::ColCtx(0), g[v], row, e0 + v,
                     p.param_c, o);
          x = outside[v] ? outv[v] : x;
          if (TABLE) {
            const int col = e0 + v;
            if (col >= j0 && col < j0 + BW && col < W)
              static_cast<typename F::OutT*>(p.table)[row * p.table_pitch + col] = o;
          }
          nw[v] = x;
        }
#pragma unroll
        for (int v = 0; v < VP; ++v) cur[v] = nw[v];
      }
      // publish the block's bottom row (or the outputs for the last band)
      const bool last_band = (b == nbands - 1);
      if (!last_band) {
        T* dst = bring + (int64_t)(b % kPrevRing) * p.bnd_stride;
#pragma unroll
        for (int v = 0; v < VP; ++v) {
          const int col = e0 + v;
          if (col >= j0 && col < j0 + BW && col < W) __stcg(dst + col, cur[v]);
        }
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
      if (lane == 0 && p.trace != nullptr && J < p.trace_chunks)
        p.trace[((int64_t)b * p.trace_chunks + J) * 2 + 1] = globaltimer_ns();
      // advance: every row of t_cur has been issued, so t_nxt has been claimed
      t_cur = t_nxt;
      t_nxt = -1;
      iss = 0;
      if (iss_done) {   // the issue cursor already finished the new t_cur: move it on
        iss_done = false;
        iss = 1;
        ir = 0;
        t_nxt = claim();
        set_issue_task(t_nxt);
      }
    }
  }
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

template <class F>
static cudaError_t launch_pr(const FillParams& p, int grid, cudaStream_t s) {
  if (p.block_cols == -1) {   // TMA path requested by the planner
    const int g = grid * kPrevWarps / kPrTmaWarps;
    constexpr int VP = kPrevV + 2 * kPrevBandRows / 32;
    const size_t smem = sizeof(typename F::GridT) * kPrTmaWarps * kPrRing * 32 * VP +
                        sizeof(uint64_t) * kPrTmaWarps * kPrRing;
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(prevrow_tma_kernel<F, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      cudaFuncSetAttribute(prevrow_tma_kernel<F, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      attr = true;
    }
    if (p.table != nullptr)
      prevrow_tma_kernel<F, true><<<g, kPrTmaWarps * 32, smem, s>>>(p);
    else
      prevrow_tma_kernel<F, false><<<g, kPrTmaWarps * 32, smem, s>>>(p);
    return cudaGetLastError();
  }
  if (p.table != nullptr)
    prevrow_kernel<F, true><<<grid, kPrevWarps * 32, 0, s>>>(p);
  else
    prevrow_kernel<F, false><<<grid, kPrevWarps * 32, 0, s>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_prevrow(int func, const FillParams& p, int grid, cudaStream_t s) {
  switch (func) {
    case 3: return launch_pr<CellMinPath3>(p, grid, s);
    case 4: return launch_pr<CellDiagMaxPlus>(p, grid, s);
    case 5: return launch_pr<CellMin2Plus>(p, grid, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace lddp
