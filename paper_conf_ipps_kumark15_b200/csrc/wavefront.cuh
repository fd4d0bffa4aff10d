// wavefront.cuh -- persistent strip-wavefront kernel for the Anti-diagonal (t = i + j) and
// Knight-Move (t = 2i + j) categories (Fig. 2 [L117-L122]; §III.A [L148-L168], §III.D
// [L217-L241]).  One launch per fill; no launch per diagonal (the paper's K1/K4, [L150]).
//
// Decomposition:
//  * The table is cut into horizontal STRIPS of SH = W*32*R rows, bottom-aligned so the last
//    strip ends at row m-1 (strip 0 may start above row 0; its virtual row -1 is overridden
//    with the initialisation, rows above that are don't-care).  Persistent CTAs claim strips in
//    increasing order with an atomic counter, so every strip waits only on a strip that an
//    already-running CTA owns (deadlock-free without co-residency).
//  * Inside a CTA, W compute warps form a systolic array of 32*W lanes; lane g owns R rows.
//    Row r of lane k in warp w processes column  c = tau - k*D - r*SIG  at warp-local step tau,
//    D = R*SIG + E.  SIG = 0/1: anti-diagonal (row r+1 needs U of row r at the same / previous
//    step), SIG = 2: knight-move (UR of the row above must be one step old).  E >= 1 extra
//    steps of lag give the shuffle latency slack.  L, UL, U, UR of rows inside a lane come from
//    a per-row register history; row 0 gets the row above from lane k-1 through one
//    __shfl_sync per step into a register FIFO (lane 0 gets it from lane 31, which injects the
//    warp's top-link value: a rotate-by-one shuffle).
//  * Warps hand their bottom row to the next warp through shared-memory LINKS: rings of NS
//    chunks of C = 32 entries (value + column context) guarded by full/empty mbarriers.
//    Link 0 is fed by a LOADER warp from the previous strip's boundary row in global memory
//    (epoch-tagged release/acquire progress flag per 32 columns); link W is drained by a
//    STORER warp into this strip's boundary row (or into last_row / score for the last strip).
//  * The DP table is virtual: only boundary rows (L2-resident) and requested outputs touch
//    global memory.
#pragma once
#include <cstdint>
#include "cellfn.cuh"
#include "params.h"
#include "sync.cuh"

namespace lddp {

constexpr int kChunk = 32;  // link chunk = 32 entries = one per lane

template <class F>
struct LinkEntry {
  typename F::T v;
  typename F::ColCtx cc;
};

template <class F, int R, int SIG, int E, int W, bool TABLE>
struct Wave {
  using T = typename F::T;
  using CC = typename F::ColCtx;
  using RC = typename F::RowCtx;
  using G = typename F::GridT;
  using O = typename F::OutT;
  using Entry = LinkEntry<F>;
  static constexpr int C = kChunk;
  static constexpr int D = R * SIG + E;      // per-lane lag in steps
  static constexpr int NS = 8;               // ring slots per link
  static constexpr int HV = SIG + 1;         // value history depth per row
  static constexpr int HC = SIG > 0 ? SIG : 1;  // column-context history depth per row
  static constexpr int FV = SIG + E + 1;     // FIFO depth (values from the lane above)
  static constexpr int FC = SIG + E;         // FIFO depth (column contexts)
  static constexpr int kThreads = (W + 2) * 32;
  static constexpr int TAU0 = -32 - SIG - E; // step at which lane 31 injects top entry q = 0
  static_assert(E >= 1, "need at least one step of shuffle slack");
  static_assert(SIG >= 2 || !(F::kMask & NB_UR), "UR needs the knight-move skew (SIG = 2)");
  static_assert(SIG + E >= 2 || !(F::kMask & NB_UR), "UR of row 0 must be at least one step old");

  struct Smem {
    Entry link[W + 1][NS][C];
    uint64_t full[W + 1][NS];
    uint64_t empty[W + 1][NS];
    uint64_t bar;        // CTA barrier (abort-aware)
    int strip;
  };
};

// CTA-wide barrier built on an mbarrier so that a watchdog abort can never leave a warp parked
// in bar.sync.  `phase` is the per-thread running parity.
__device__ __forceinline__ bool cta_sync(uint64_t* bar, uint32_t& phase, Control* ctl,
                                         uint64_t timeout_ns) {
  mbar_arrive(bar);
  bool ok = mbar_wait(bar, phase, ctl, timeout_ns);
  phase ^= 1u;
  return ok;
}

template <class F, int R, int SIG, int E, int W, bool TABLE>
struct WaveCompute {
  using WV = Wave<F, R, SIG, E, W, TABLE>;
  using T = typename WV::T;
  using CC = typename WV::CC;
  using RC = typename WV::RC;
  using G = typename WV::G;
  using O = typename WV::O;
  using Entry = typename WV::Entry;
  static constexpr int C = WV::C, D = WV::D, HV = WV::HV, HC = WV::HC, FV = WV::FV, FC = WV::FC;

  T hist[R][HV];   // hist[r][d] = value of row r at step tau-1-d
  CC hcc[R][HC];   // hcc[r][d]  = column context of row r at step tau-1-d
  T fifo[FV];      // fifo[d]    = value received from the lane above at the end of step tau-1-d
  CC fcc[FC > 0 ? FC : 1];
  RC rc[R];
  int64_t irow[R];

  template <bool CHECKED>
  __device__ __forceinline__ void chunk(const FillParams& p, const int lane, const int tau_k,
                                        const Entry* __restrict__ top, Entry* __restrict__ bot,
                                        const bool has_bot) {
    const int n = p.cols;
    const int lane_off = lane * D;
#pragma unroll
    for (int st = 0; st < C; ++st) {
      const int tau = tau_k + st;
      T nw[R];
      CC ncc[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int c = tau - lane_off - r * SIG;
        T L = hist[r][0], U, UL, UR;
        CC cc;
        if (r == 0) {
          U = fifo[SIG + E - 1];
          UL = fifo[SIG + E];
          UR = fifo[(SIG + E >= 2) ? SIG + E - 2 : 0];
          cc = fcc[SIG + E - 1];
        } else {
          if (SIG == 0) {
            U = nw[r - 1];
            cc = ncc[r - 1];
          } else {
            U = hist[r - 1][SIG > 0 ? SIG - 1 : 0];
            cc = hcc[r - 1][SIG > 0 ? SIG - 1 : 0];
          }
          UL = hist[r - 1][SIG];
          UR = hist[r - 1][SIG >= 2 ? SIG - 2 : 0];
        }
        G g = G(0);
        if (F::kGridIn) {
          if (CHECKED) {
            if (c >= 0 && c < n && irow[r] >= 0) g = F::load(p, irow[r], c);
          } else {
            g = F::load(p, irow[r], c);
          }
        }
        O o;
        T v = F::f(L, UL, U, UR, rc[r], cc, g, irow[r], c + p.col0, p.param_c, o);
        if (CHECKED) {
          if (c == -1) {
            if (p.lcol_in != nullptr) {
              if (irow[r] >= 0) v = __ldcg(static_cast<const T*>(p.lcol_in) + irow[r]);
            } else {
              v = F::left(p, irow[r]);
            }
          }
          if (c == n) v = F::right(p, irow[r]);
          if (irow[r] == -1) v = F::top(p, c + p.col0);
          if (c >= 0 && c < n && irow[r] >= 0) {
            if (TABLE) static_cast<O*>(p.table)[irow[r] * p.table_pitch + c] = o;
            if (c == n - 1) {
              if (p.last_col != nullptr) static_cast<T*>(p.last_col)[irow[r]] = v;
              if (p.rcol_out != nullptr) static_cast<T*>(p.rcol_out)[irow[r]] = v;
            }
          }
        } else {
          if (TABLE) static_cast<O*>(p.table)[irow[r] * p.table_pitch + c] = o;
        }
        nw[r] = v;
        ncc[r] = cc;
      }
      // link I/O by lane 31 and the rotate-by-one shuffle
      if (has_bot && lane == 31) bot[st] = Entry{nw[R - 1], ncc[R - 1]};
      const Entry te = top[st];
      const T sv = (lane == 31) ? te.v : nw[R - 1];
      const CC scc = (lane == 31) ? te.cc : ncc[R - 1];
      const int src = (lane + 31) & 31;
      const T rv = __shfl_sync(0xffffffffu, sv, src);
      const CC rcc = __shfl_sync(0xffffffffu, scc, src);
      // shift histories
#pragma unroll
      for (int r = 0; r < R; ++r) {
#pragma unroll
        for (int d = HV - 1; d > 0; --d) hist[r][d] = hist[r][d - 1];
        hist[r][0] = nw[r];
        if (SIG > 0) {
#pragma unroll
          for (int d = HC - 1; d > 0; --d) hcc[r][d] = hcc[r][d - 1];
          hcc[r][0] = ncc[r];
        }
      }
#pragma unroll
      for (int d = FV - 1; d > 0; --d) fifo[d] = fifo[d - 1];
      fifo[0] = rv;
#pragma unroll
      for (int d = FC - 1; d > 0; --d) fcc[d] = fcc[d - 1];
      fcc[0] = rcc;
    }
  }
};

template <class F, int R, int SIG, int E, int W, bool TABLE>
__global__ void __launch_bounds__(Wave<F, R, SIG, E, W, TABLE>::kThreads)
wavefront_kernel(const FillParams p) {
  using WV = Wave<F, R, SIG, E, W, TABLE>;
  using T = typename WV::T;
  using CC = typename WV::CC;
  using Entry = typename WV::Entry;
  constexpr int C = WV::C, NS = WV::NS, D = WV::D;

  __shared__ typename WV::Smem sm;
  Control* ctl = static_cast<Control*>(p.ctl);
  const uint64_t tmo = p.timeout_ns;
  const int lane = threadIdx.x & 31;
  const int wid = threadIdx.x >> 5;
  const int n = p.cols;
  const int NQ = p.nchunks;
  const uint64_t ep = p.epoch << 32;

  if (threadIdx.x == 0) {
    for (int l = 0; l <= W; ++l)
      for (int s = 0; s < NS; ++s) {
        mbar_init(&sm.full[l][s], 1);
        mbar_init(&sm.empty[l][s], 1);
      }
    mbar_init(&sm.bar, WV::kThreads);
  }
  __syncthreads();

  uint32_t bar_phase = 0;
  uint32_t iter = 0;
  while (true) {
    if (threadIdx.x == 0) sm.strip = (int)atomicAdd(&ctl->claim, 1u);
    if (!cta_sync(&sm.bar, bar_phase, ctl, tmo)) return;
    const int s = sm.strip;
    if (s >= p.nstrips) break;
    const int64_t strip_top = p.row0 + (int64_t)s * p.strip_rows;

    if (wid < W) {
      // ------------------------------------------------------------------ compute warp
      WaveCompute<F, R, SIG, E, W, TABLE> cs;
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int64_t i = strip_top + (int64_t)(wid * 32 + lane) * R + r;
        cs.irow[r] = i;
        cs.rc[r] = (i >= 0 && i < p.rows) ? F::row_ctx(p, i) : typename WV::RC(0);
#pragma unroll
        for (int d = 0; d < WV::HV; ++d) cs.hist[r][d] = T(0);
#pragma unroll
        for (int d = 0; d < WV::HC; ++d) cs.hcc[r][d] = CC(0);
      }
#pragma unroll
      for (int d = 0; d < WV::FV; ++d) cs.fifo[d] = T(0);
#pragma unroll
      for (int d = 0; d < (WV::FC > 0 ? WV::FC : 1); ++d) cs.fcc[d] = CC(0);
      if (p.lcol_in != nullptr) {   // multi-GPU: rank g-1's right column of this strip
        if (!wait_flag<true>(p.lflag_in + s, (p.wepoch << 32) | 1u, ctl, tmo)) return;
      }
      const bool virt = strip_top < 0;
      const int K = NQ + D;
      for (int k = 0; k < K; ++k) {
        const bool has_top = k < NQ;
        const bool has_bot = k >= D;
        const uint32_t gt = iter * (uint32_t)NQ + (uint32_t)k;
        const uint32_t gb = iter * (uint32_t)NQ + (uint32_t)(k - D);
        const Entry* top = sm.link[wid][0];
        Entry* bot = sm.link[wid + 1][0];
        if (has_top) {
          if (!mbar_wait(&sm.full[wid][gt % NS], (gt / NS) & 1u, ctl, tmo)) return;
          top = sm.link[wid][gt % NS];
        }
        if (has_bot) {
          if (gb / NS >= 1) {
            if (!mbar_wait(&sm.empty[wid + 1][gb % NS], ((gb / NS) - 1) & 1u, ctl, tmo)) return;
          }
          bot = sm.link[wid + 1][gb % NS];
        }
        const int tau_k = WV::TAU0 + k * C;
        const bool steady = !virt && (tau_k - 31 * D - (R - 1) * SIG >= 0) && (tau_k + C < n);  // max column < n-1: last_col / rcol cells stay checked
        if (steady)
          cs.template chunk<false>(p, lane, tau_k, top, bot, has_bot);
        else
          cs.template chunk<true>(p, lane, tau_k, top, bot, has_bot);
        __syncwarp();
        if (lane == 0) {
          if (has_top) mbar_arrive(&sm.empty[wid][gt % NS]);
          if (has_bot) mbar_arrive(&sm.full[wid + 1][gb % NS]);
        }
      }
      if (p.rcol_out != nullptr) __threadfence_system();
    } else if (wid == W) {
      // ------------------------------------------------------------------ loader warp
      const T* prev = static_cast<const T*>(p.bnd) + (int64_t)(s - 1) * p.bnd_stride;
      for (int k = 0; k < NQ; ++k) {
        const uint32_t g = iter * (uint32_t)NQ + (uint32_t)k;
        const int slot = g % NS;
        if (g / NS >= 1) {
          if (!mbar_wait(&sm.empty[0][slot], ((g / NS) - 1) & 1u, ctl, tmo)) return;
        }
        const int q = k * C + lane;
        const int c = q - 32;
        T v;
        if (s > 0) {
          if (!wait_flag<false>(p.prog + (s - 1), ep | (uint64_t)(k + 1), ctl, tmo)) return;
          v = __ldcg(prev + q);
        } else {
          v = F::top(p, c + p.col0);
        }
        CC cc = (c >= 0 && c < n) ? F::col_ctx(p, c + p.col0) : CC(0);
        sm.link[0][slot][lane] = Entry{v, cc};
        __syncwarp();
        if (lane == 0) mbar_arrive(&sm.full[0][slot]);
      }
    } else {
      // ------------------------------------------------------------------ storer warp
      const bool last = (s == p.nstrips - 1);
      T* mine = static_cast<T*>(p.bnd) + (int64_t)s * p.bnd_stride;
      T rmin = T(0);
      bool have = false;
      for (int k = 0; k < NQ; ++k) {
        const uint32_t g = iter * (uint32_t)NQ + (uint32_t)k;
        const int slot = g % NS;
        if (!mbar_wait(&sm.full[W][slot], (g / NS) & 1u, ctl, tmo)) return;
        const T v = sm.link[W][slot][lane].v;
        __syncwarp();
        if (lane == 0) mbar_arrive(&sm.empty[W][slot]);
        const int q = k * C + lane;
        const int c = q - 32;
        if (!last) {
          __stcg(mine + q, v);
          __threadfence();
          __syncwarp();
          if (lane == 0) st_release_gpu(p.prog + s, ep | (uint64_t)(k + 1));
        } else if (c >= 0 && c < n) {
          if (p.last_row != nullptr) static_cast<T*>(p.last_row)[c] = v;
          if (F::kScore == SCORE_LAST_CELL && c == n - 1 && p.score != nullptr && p.is_last_rank)
            *static_cast<T*>(p.score) = v;
          if (F::kScore == SCORE_ROW_MIN) {
            rmin = have ? min(rmin, v) : v;
            have = true;
          }
        }
      }
      if (F::kScore == SCORE_ROW_MIN && last && p.score != nullptr) {
        for (int off = 16; off > 0; off >>= 1) {
          const T o = __shfl_xor_sync(0xffffffffu, rmin, off);
          const bool oh = __shfl_xor_sync(0xffffffffu, have ? 1 : 0, off) != 0;
          if (oh) rmin = have ? min(rmin, o) : o;
          have = have || oh;
        }
        if (lane == 0) *static_cast<T*>(p.score) = rmin;
      }
    }
    // end of strip: publish the right column to rank g+1 (multi-GPU), recycle the CTA
    if (!cta_sync(&sm.bar, bar_phase, ctl, tmo)) return;
    if (p.rflag_out != nullptr && threadIdx.x == 0) {
      __threadfence_system();
      st_release_sys(p.rflag_out + s, (p.wepoch << 32) | 1u);
    }
    ++iter;
  }
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned d = atomicAdd(&ctl->done, 1u);
    if (d == gridDim.x - 1) {
      atomicExch(&ctl->claim, 0u);
      atomicExch(&ctl->done, 0u);
    }
  }
}

}  // namespace lddp
