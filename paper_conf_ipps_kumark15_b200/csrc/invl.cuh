// invl.cuh -- Inverted-L category kernel ("the remaining pattern", t = min(i,j)) [L197-L215],
// Fig. 2(c), contributing set {UL} (Table I [L129], [L203]).
//
// With UL as the only dependency, every diagonal d = j - i is an independent chain.  The paper
// processes shrinking inverted-L shells with one launch each [L205] and notes the horizontal
// case-1 schedule is better for coalescing [L215], [L296-L298].  On B200 the natural form is
// neither: one lane per diagonal chain, 32 adjacent diagonals per warp, walking rows in
// lockstep -- so lane l touches column i + d0 + l of row i: every row step is one coalesced
// 128-byte load (and store), no inter-thread dependency at all: pure HBM streaming.
//
// The time of the fill is the time of the longest chains (min(H, W) rows), so each warp keeps
// kInvlDepth rows of loads in flight (two register blocks: the next block is loaded while the
// current one is evaluated): 2048 warps x 64 rows x 128 B = 16 MB in flight for C6, enough to
// cover the HBM latency at full bandwidth.  Every warp owns one group of 32
// diagonals for the whole fill (the grid holds all of them: no tail of late-starting chains).
#pragma once
#include <cstdint>
#include "cellfn.cuh"
#include "params.h"
#include "sync.cuh"

namespace lddp {

constexpr int kInvlWarps = 4;
constexpr int kInvlBlock = 16;   // rows per register block (two blocks in flight; 16 keeps every warp resident: C6 2.70 -> 2.19 ms against 32)

// F::kDirectGrid (the compiled-in f's): the per-cell input is element (i, j) of p.grid, read
// with a running pointer (and mirrored columns); otherwise (user functors, include/lddp_user.cuh)
// through F::load.
template <class F, class = void>
struct InvlDirect { static constexpr bool value = false; };
template <class F>
struct InvlDirect<F, decltype(void(F::kDirectGrid))> { static constexpr bool value = F::kDirectGrid; };

// MIRROR: the kernel's column j' is the grid's column W-1-j' (mInverted-L twin, {UR} -> {UL}).
template <class F, bool TABLE, bool MIRROR, int BLK = kInvlBlock>
__global__ void __launch_bounds__(kInvlWarps * 32) invl_kernel(const FillParams p) {
  using T = typename F::T;
  using G = typename F::GridT;
  static_assert(F::kMask == NB_UL, "inverted-L category: contributing set must be {UL}");
  const int lane = threadIdx.x & 31;
  const int64_t H = p.rows;
  const int W = p.cols;
  // this launch's diagonals d = j - i in [diag_lo, diag_hi) (all of [-(H-1), W-1] on one GPU;
  // a contiguous share per rank for lddp_fill_multi: the chains are independent, no exchange)
  const int64_t dlo0 = p.diag_lo, dhi0 = p.diag_hi;
  const int64_t nwarps_total = (dhi0 - dlo0 + 31) / 32;
  const int64_t gw0 = (int64_t)blockIdx.x * kInvlWarps + (threadIdx.x >> 5);
  const int64_t gstride = (int64_t)gridDim.x * kInvlWarps;
  for (int64_t gw = gw0; gw < nwarps_total; gw += gstride) {
    const int64_t d = dlo0 + gw * 32 + lane;         // this lane's diagonal
    const bool live = d < dhi0;
    // rows this warp visits: union of its lanes' chains
    const int64_t dlo = dlo0 + gw * 32;
    const int64_t dhi = min(dhi0 - 1, dlo + 31);
    const int64_t ibeg = max((int64_t)0, -dhi);
    const int64_t iend = min(H, (int64_t)W - dlo);   // exclusive
    // this lane's chain: rows [ia, ib)
    const int64_t ia = max((int64_t)0, -d), ib = min(H, (int64_t)W - d);
    // element (i, i + d) = src + i * step (mirrored: grid column W-1-(i+d))
    const G* src = static_cast<const G*>(p.grid) + (MIRROR ? (int64_t)W - 1 - d : d);
    const int64_t step = MIRROR ? p.grid_pitch - 1 : p.grid_pitch + 1;
    // UL of the chain's first cell: the row above row 0 (d >= 0) or the column left of column 0
    T v = MIRROR ? T(0) : (d >= 0 ? F::top(p, (int)d - 1 + p.col0) : F::left(p, -d - 1));
    G cur[BLK], nxt[BLK];
    auto load_block = [&](G* dst, int64_t i0) {
#pragma unroll
      for (int u = 0; u < BLK; ++u) {
        const int64_t i = i0 + u;
        if constexpr (InvlDirect<F>::value)
          dst[u] = (live && i >= ia && i < ib) ? __ldcs(src + i * step) : G(0);
        else
          dst[u] = (live && i >= ia && i < ib) ? F::load(p, i, (int)(i + d)) : G(0);
      }
    };
    load_block(cur, ibeg);
    for (int64_t i0 = ibeg; i0 < iend; i0 += BLK) {
      if (i0 + BLK < iend) load_block(nxt, i0 + BLK);
      // whole block inside every lane's chain and short of the last row / column: no per-cell
      // range or output tests (i, j are still passed to f: a user f may read them)
      const bool inner = live && i0 >= ia && i0 + BLK < ib && i0 + BLK < H;
      if (__all_sync(0xffffffffu, inner)) {
#pragma unroll
        for (int u = 0; u < BLK; ++u) {
          const int64_t i = i0 + u;
          const int64_t j = i + d;
          typename F::OutT o;
          v = F::f(v, v, v, v, typename F::RowCtx(0), typename F::ColCtx(0), cur[u], i,
                   (int)j + p.col0, p.param_c, o);
          if (TABLE) static_cast<typename F::OutT*>(p.table)[i * p.table_pitch + (MIRROR ? (int64_t)W - 1 - j : j)] = o;
        }
#pragma unroll
        for (int u = 0; u < BLK; ++u) cur[u] = nxt[u];
        continue;
      }
#pragma unroll
      for (int u = 0; u < BLK; ++u) {
        const int64_t i = i0 + u;
        const int64_t j = i + d;
        if (live && i >= ia && i < ib) {
          typename F::OutT o;
          v = F::f(v, v, v, v, typename F::RowCtx(0), typename F::ColCtx(0), cur[u], i,
                   (int)j + p.col0, p.param_c, o);
          const int64_t jg = MIRROR ? (int64_t)W - 1 - j : j;   // the grid's column
          if (TABLE) static_cast<typename F::OutT*>(p.table)[i * p.table_pitch + jg] = o;
          if (i == H - 1 && p.last_row != nullptr) static_cast<T*>(p.last_row)[jg] = v;
          if (j == W - 1 && p.last_col != nullptr) static_cast<T*>(p.last_col)[i] = v;
        }
      }
#pragma unroll
      for (int u = 0; u < BLK; ++u) cur[u] = nxt[u];
    }
  }
}

}  // namespace lddp
