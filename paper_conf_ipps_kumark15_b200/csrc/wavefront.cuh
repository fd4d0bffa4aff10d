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
#include <cstring>
#include "cellfn.cuh"
#include "params.h"
#include "sync.cuh"

namespace lddp {

constexpr int kChunk = 32;  // link chunk = 32 entries = one per lane
constexpr int kUnroll = 8;  // steps per unrolled loop body
constexpr int kBatch = 4;   // chunks moved per loader / storer round trip
constexpr int kBRing = 4096; // column-context ring (entries); index = (column + 32) & (kBRing - 1)
constexpr int kGridPrefetchCols = 256;  // L1 prefetch distance of grid rows (columns)


template <class F, class = void>
struct ByteIO { static constexpr bool value = false; };
template <class F>
struct ByteIO<F, decltype(void(F::kByteIO))> { static constexpr bool value = F::kByteIO; };

template <class F, int R, int SIG, int E, int W, bool TABLE, int GS = (SIG == 0 ? R : 1)>
struct Wave {
  using T = typename F::T;
  using CC = typename F::ColCtx;
  using RC = typename F::RowCtx;
  using G = typename F::GridT;
  using O = typename F::OutT;
  static constexpr int C = kChunk;
  static constexpr int NG = R / GS;          // row groups per lane (rows chained within a group)
  static constexpr int D = NG * SIG + E;     // per-lane lag in steps
  static constexpr int NS = 16;              // ring slots per link
  static constexpr int HV = SIG + 1;         // value history depth per row
  static constexpr int HC = SIG > 0 ? SIG : 1;  // column-context history depth per row
  static constexpr int FV = SIG + E + 1;     // FIFO depth (values from the lane above)
  static constexpr int kThreads = (W + 2) * 32;
  static constexpr int TAU0 = -32 - SIG - E; // step at which lane 31 injects top entry q = 0
  static_assert(E >= 1, "need at least one step of shuffle slack");
  static_assert(R % GS == 0, "row groups must tile the lane's rows");
  static_assert(GS == 1 || SIG <= 1 || !(F::kMask & NB_UR), "UR needs every row skewed (GS = 1)");
  static_assert(SIG >= 2 || !(F::kMask & NB_UR), "UR needs the knight-move skew (SIG = 2)");
  static_assert(SIG + E >= 2 || !(F::kMask & NB_UR), "UR of row 0 must be at least one step old");

  struct Smem {
    alignas(16) T link[W + 1][NS][C];
    uint64_t full[W + 1][NS];
    uint64_t empty[W + 1][NS];
    typename F::ColCtx bring[F::kGridIn ? 32 : kBRing];   // column contexts staged by the loader
    // byte-image f's (FS): per compute warp, 3 chunks of 32 row segments x 32 bytes of input and
    // one chunk of output, rows padded to 9 words (conflict-free lane-row reads)
    uint32_t stg_in[ByteIO<F>::value ? W : 1][ByteIO<F>::value ? 3 * 32 * 9 : 1];
    uint32_t stg_out[ByteIO<F>::value ? W : 1][ByteIO<F>::value ? 32 * 9 : 1];
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

template <class T>
__device__ __forceinline__ T bits_to(uint32_t x) {
  T t;
  memcpy(&t, &x, sizeof(T));
  return t;
}
template <class T>
__device__ __forceinline__ uint32_t to_bits(T t) {
  uint32_t x;
  memcpy(&x, &t, sizeof(T));
  return x;
}

template <class F, int R, int SIG, int E, int W, bool TABLE, int GS = (SIG == 0 ? R : 1)>
struct WaveCompute {
  using WV = Wave<F, R, SIG, E, W, TABLE, GS>;
  using T = typename WV::T;
  using CC = typename WV::CC;
  using RC = typename WV::RC;
  using G = typename WV::G;
  using O = typename WV::O;
  static constexpr int C = WV::C, D = WV::D, HV = WV::HV, HC = WV::HC, FV = WV::FV, NG = WV::NG;
  static_assert(sizeof(T) == 4, "link values are 32-bit");
  // uint8 image in / out as aligned 32-bit words: every lane-row's column must share the step's
  // residue mod 4 (R = 1 and D % 4 == 0), and chunk starts are multiples of 4.
  static constexpr bool kVec = ByteIO<F>::value && R == 1 && (D % 4 == 0) && ((WV::TAU0 % 4) == 0);

  T hist[R][HV];   // hist[r][d] = value of row r at step tau-1-d
  CC hcc[R][HC];   // hcc[r][d]  = column context of row r at step tau-1-d (SIG > 0)
  T fifo[FV];      // fifo[d]    = value received from the lane above at the end of step tau-1-d
  RC rc[R];
  int irow[R];     // global row of each lane-row (may be < 0 in strip 0: virtual rows)
  T leftv[R];      // value of column -1 of the row (initialisation, or rank g-1's column)
  T rightv[R];     // value of column n of the row (only read through UR)
  bool vtop[R];    // the lane-row is strip 0's virtual row -1 (holds the top initialisation)
  bool rvalid[R];  // 0 <= row < m
  T rlast[R];      // the row's value at column n-1 (captured in boundary chunks)
  G gA[R][kUnroll], gB[R][kUnroll];   // grid prefetch pipeline (kGridIn f's)
  uint32_t* stg_in;    // this warp's input staging [3][32][9] words (kVec)
  uint32_t* stg_out;   // this warp's output staging [32][9] words (kVec)
  int row_base;        // global row of lane 0's row 0
  int carry_tau;   // chunk start whose first two sub-blocks gA / gB hold (else invalid)

  // Byte-image staging (kVec: R = 1, D = 4): lane-row rho's 32 input bytes of the chunk that
  // starts at step tau are the columns [tau - rho*D, tau - rho*D + 32) -- 8 aligned words.  The
  // warp copies them cooperatively, 8 lanes per row segment (4 segments per instruction, so
  // each instruction touches 4 lines instead of 32), with cp.async two chunks ahead.
  __device__ __forceinline__ void stage_load(const FillParams& p, const int lane, const int tau) const {
    const int n = p.cols;
    const int k = (tau - WV::TAU0) / C;
    const uint8_t* grid = static_cast<const uint8_t*>(p.grid);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int rho = 4 * i + (lane >> 3);
      const int j = lane & 7;
      const int col = tau - rho * D + 4 * j;
      const int row = row_base + rho;
      const bool ok = row >= 0 && row < p.rows && col >= 0 && col < n;   // row padded to 4 B
      cp_async_4(&stg_in[((k % 3) * 32 + rho) * 9 + j], ok ? grid + (int64_t)row * p.grid_pitch + col : grid,
                 ok ? 4u : 0u);
    }
    cp_async_commit();
  }
  // Cooperative store of the chunk's output bytes (packed by their lane-rows in stg_out).
  __device__ __forceinline__ void stage_store(const FillParams& p, const int lane, const int tau) const {
    const int n = p.cols;
    uint8_t* out = static_cast<uint8_t*>(p.table);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int rho = 4 * i + (lane >> 3);
      const int j = lane & 7;
      const int col = tau - rho * D + 4 * j;
      const int row = row_base + rho;
      if (row < 0 || row >= p.rows) continue;
      const uint32_t w = stg_out[rho * 9 + j];
      uint8_t* rp = out + (int64_t)row * p.table_pitch;
      if (col >= 0 && col + 3 < n) {
        *reinterpret_cast<uint32_t*>(rp + col) = w;
      } else if (col + 3 >= 0 && col < n) {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (col + q >= 0 && col + q < n) rp[col + q] = (uint8_t)(w >> (8 * q));
      }
    }
  }

  // Loads for the 8 steps starting at tau0: row 0's column context and each row's grid input.
  const CC* bring;  // shared-memory column-context ring (staged by the loader warp)

  template <int MODE, int U>
  __device__ __forceinline__ void prefetch(const FillParams& p, const int lane_off, const int tau0,
                                           CC (&cc)[U], G (&g)[R][U]) const {
    const int n = p.cols;
#pragma unroll
    for (int su = 0; su < U; ++su) {
      const int c0 = tau0 + su - lane_off;
      cc[su] = F::kGridIn ? CC(0) : bring[(c0 + 32) & (kBRing - 1)];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int c = c0 - (r / GS) * SIG;
        if constexpr (kVec) {
          if (su % 4 == 0) {
            // one staged word covers this step and the next three (see stage_load)
            const int k = (tau0 - WV::TAU0) / C;            // chunk index of this sub-block
            const int w = ((tau0 - WV::TAU0) % C + su) / 4;  // word within the lane-row segment
            const uint32_t wd = stg_in[((k % 3) * 32 + lane_off / D) * 9 + w];
#pragma unroll
            for (int q = 0; q < 4; ++q)
              if (su + q < U) g[r][su + q] = F::from_byte((wd >> (8 * q)) & 0xffu);
          }
          continue;
        }
        if (!F::kGridIn) {
          g[r][su] = G(0);
        } else if (MODE == 2) {
          g[r][su] = (rvalid[r] && (unsigned)c < (unsigned)n) ? F::load(p, irow[r], c) : G(0);
        } else if (MODE == 1) {
          g[r][su] = rvalid[r] ? F::load(p, irow[r], c) : G(0);
        } else {
          g[r][su] = F::load(p, irow[r], c);
        }
      }
    }
  }

  // One chunk of C steps.  MODE 0: steady (every cell interior); MODE 1: steady + strip 0's
  // virtual row -1 (one select per cell); MODE 2: checked (boundary columns, virtual rows,
  // output columns).
  // Per step: R cells, one __shfl_sync (the bottom row value, lane k -> k+1, lane 31 -> 0
  // injecting the warp's top link), one L1-cached load of row 0's column context.  Lane 31's
  // top-link values and bottom-link values move 8 steps at a time as two 128-bit smem ops.
  template <int MODE>
  __device__ __forceinline__ void chunk(const FillParams& p, const int lane, const int tau_k,
                                        const T* __restrict__ top, T* __restrict__ bot,
                                        const bool has_bot) {
    // the checked body is executed only a few chunks per strip: keep its code small
    constexpr int U = kUnroll;
    constexpr bool CHECKED = MODE == 2;
    const int n = p.cols;
    const int lane_off = lane * D;
    // Row 0's column contexts and every row's grid inputs are loaded one 8-step block ahead,
    // so the L1 / L2 latency of those loads is off the per-step critical path.
    CC ccc[U];
    G gcur[R][U];
    if (F::kGridIn) {
      // pull each lane-row's grid line 256 columns ahead into L1 (the per-cell loads of the
      // next chunks then hit L1; an image row is streamed once per lane-row)
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int c = tau_k - lane_off - (r / GS) * SIG + kGridPrefetchCols;
        if (rvalid[r] && c >= 0 && c < n) F::prefetch_l1(p, irow[r], c);
      }
    }
    // Grid inputs (image / cost rows) stream from DRAM: they are kept two sub-blocks ahead in
    // a register pipeline (gA, gB) that also carries across chunk boundaries; the loads are
    // always bounds-guarded so a carried value is valid whatever the next chunk's mode.
    // Column contexts come from the shared-memory ring one sub-block ahead.
    constexpr bool kDeep = F::kGridIn && !kVec;
    if constexpr (kVec) {
      stage_load(p, lane, tau_k + 2 * C);   // two chunks ahead
      cp_async_wait_group<2>();             // this chunk's segments have landed (own copies)
      __syncwarp();                         // ... and every lane's copies are visible
    }
    if (kDeep) {
      if (carry_tau != tau_k) {
        prefetch<2, U>(p, lane_off, tau_k, ccc, gA);
        prefetch<2, U>(p, lane_off, tau_k + U, ccc, gB);
      }
    }
    prefetch<MODE, U>(p, lane_off, tau_k, ccc, gcur);
#pragma unroll 1
    for (int sb = 0; sb < C; sb += U) {
      CC ccn[U];
      G gnxt[R][U];
      if (kDeep) {
#pragma unroll
        for (int su = 0; su < U; ++su)
#pragma unroll
          for (int r = 0; r < R; ++r) {
            gcur[r][su] = gA[r][su];
            gA[r][su] = gB[r][su];
          }
        prefetch<2, U>(p, lane_off, tau_k + sb + 2 * U, ccn, gB);
        if (sb + U < C) prefetch<MODE, U>(p, lane_off, tau_k + sb + U, ccn, gnxt);
      } else {
        if (sb + U < C) prefetch<MODE, U>(p, lane_off, tau_k + sb + U, ccn, gnxt);
      }
      T tv[U];
      if (U == 8) {
        const uint4 q0 = reinterpret_cast<const uint4*>(top + sb)[0];
        const uint4 q1 = reinterpret_cast<const uint4*>(top + sb)[1];
        tv[0] = bits_to<T>(q0.x); tv[1 % U] = bits_to<T>(q0.y); tv[2 % U] = bits_to<T>(q0.z); tv[3 % U] = bits_to<T>(q0.w);
        tv[4 % U] = bits_to<T>(q1.x); tv[5 % U] = bits_to<T>(q1.y); tv[6 % U] = bits_to<T>(q1.z); tv[7 % U] = bits_to<T>(q1.w);
      } else {
#pragma unroll
        for (int su = 0; su < U; ++su) tv[su] = top[sb + su];
      }
      T bv[U];
      uint32_t owd = 0;   // packed output bytes (kVec)
#pragma unroll
      for (int su = 0; su < U; ++su) {
        const int tau = tau_k + sb + su;
        T nw[R];
        CC ncc[R];
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int c = tau - lane_off - (r / GS) * SIG;
          T L = hist[r][0], U, UL, UR;
          CC cc;
          if (r == 0) {
            U = fifo[SIG + E - 1];
            UL = fifo[SIG + E];
            UR = fifo[(SIG + E >= 2) ? SIG + E - 2 : 0];
            cc = ccc[su];
          } else if (SIG == 0 || r % GS != 0) {
            // inside a row group: the row above is at the same column this step
            U = nw[r - 1];
            cc = ncc[r - 1];
            UL = hist[r - 1][0];
            UR = U;   // unused (UR needs GS = 1)
          } else {
            // first row of a skewed group: the row above is SIG steps ahead
            U = hist[r - 1][SIG > 0 ? SIG - 1 : 0];
            cc = hcc[r - 1][SIG > 0 ? SIG - 1 : 0];
            UL = hist[r - 1][SIG];
            UR = hist[r - 1][SIG >= 2 ? SIG - 2 : 0];
          }
          const G g = gcur[r][su];
          O o;
          T v = F::f(L, UL, U, UR, rc[r], cc, g, irow[r], c + p.col0, p.param_c, o);
          if (CHECKED) {
            // select-only fixups: boundary columns, virtual row; the right column is captured
            // in registers (stored once per strip)
            v = (c == -1) ? leftv[r] : v;
            if (F::kMask & NB_UR) v = (c == n) ? rightv[r] : v;
            if (vtop[r]) v = F::top(p, c + p.col0);
            rlast[r] = (c == n - 1) ? v : rlast[r];
            if constexpr (kVec) {
              // packed into this lane-row's output segment; stored cooperatively per chunk
              const uint32_t ob = (uint32_t)o;
              owd = (su % 4 == 0) ? ob : (owd | (ob << (8 * (su % 4))));
              if (su % 4 == 3) stg_out[lane * 9 + (sb + su) / 4] = owd;
            } else if (TABLE && rvalid[r] && (unsigned)c < (unsigned)n) {
              static_cast<O*>(p.table)[(int64_t)irow[r] * p.table_pitch + c] = o;
            }
          } else {
            if (MODE == 1 && vtop[r]) v = F::top(p, c + p.col0);
            if constexpr (kVec) {
              const uint32_t ob = (uint32_t)o;
              owd = (su % 4 == 0) ? ob : (owd | (ob << (8 * (su % 4))));
              if (su % 4 == 3) stg_out[lane * 9 + (sb + su) / 4] = owd;
            } else if (TABLE && (MODE == 0 || rvalid[r])) {
              static_cast<O*>(p.table)[(int64_t)irow[r] * p.table_pitch + c] = o;
            }
          }
          nw[r] = v;
          ncc[r] = cc;
        }
        bv[su] = nw[R - 1];
        const T sv = (lane == 31) ? tv[su] : nw[R - 1];
        const T rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
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
      }
#pragma unroll
      for (int su = 0; su < U; ++su) {
        ccc[su] = ccn[su];
        if (!kDeep) {
#pragma unroll
          for (int r = 0; r < R; ++r) gcur[r][su] = gnxt[r][su];
        }
      }
      if (has_bot && lane == 31) {
        if (U == 8) {
          uint4* b4 = reinterpret_cast<uint4*>(bot + sb);
          b4[0] = make_uint4(to_bits(bv[0]), to_bits(bv[1 % U]), to_bits(bv[2 % U]), to_bits(bv[3 % U]));
          b4[1] = make_uint4(to_bits(bv[4 % U]), to_bits(bv[5 % U]), to_bits(bv[6 % U]), to_bits(bv[7 % U]));
        } else {
#pragma unroll
          for (int su = 0; su < U; ++su) bot[sb + su] = bv[su];
        }
      }
    }
    if (kDeep) carry_tau = tau_k + C;   // gA / gB now hold the next chunk's first two sub-blocks
    if constexpr (kVec) {
      if (TABLE) {
        __syncwarp();
        stage_store(p, lane, tau_k);
        __syncwarp();
      }
    }
  }
};

// Debug trace: stamp[0] = wait satisfied, stamp[1] = chunk done, per (strip, warp, chunk).
__device__ __forceinline__ void trace_stamp(const FillParams& p, int s, int wid, int nwarps, int k,
                                            int which) {
  if (p.trace != nullptr && k < p.trace_chunks) {
    const int64_t idx = (((int64_t)s * nwarps + wid) * p.trace_chunks + k) * 2 + which;
    p.trace[idx] = globaltimer_ns();
  }
}

template <class F, int R, int SIG, int E, int W, bool TABLE, int GS = (SIG == 0 ? R : 1)>
__global__ void __launch_bounds__(Wave<F, R, SIG, E, W, TABLE, GS>::kThreads)
wavefront_kernel(const FillParams p) {
  using WV = Wave<F, R, SIG, E, W, TABLE, GS>;
  using T = typename WV::T;
  using CC = typename WV::CC;
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
      WaveCompute<F, R, SIG, E, W, TABLE, GS> cs;
      cs.bring = sm.bring;
      cs.carry_tau = INT_MIN;
      cs.stg_in = sm.stg_in[ByteIO<F>::value ? wid : 0];
      cs.stg_out = sm.stg_out[ByteIO<F>::value ? wid : 0];
      cs.row_base = (int)(strip_top + (int64_t)wid * 32 * R);
      if (p.lcol_in != nullptr) {   // multi-GPU: rank g-1's right column of this strip
        if (!wait_flag<true>(p.lflag_in + s, (p.wepoch << 32) | 1u, ctl, tmo)) return;
      }
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int64_t i = strip_top + (int64_t)(wid * 32 + lane) * R + r;
        cs.irow[r] = (int)i;
        cs.rvalid[r] = i >= 0 && i < p.rows;
        cs.vtop[r] = i == -1;
        cs.rc[r] = cs.rvalid[r] ? F::row_ctx(p, i) : typename WV::RC(0);
        cs.rlast[r] = T(0);
        if (cs.vtop[r]) {
          cs.leftv[r] = F::top(p, p.col0 - 1);          // corner
          cs.rightv[r] = F::top(p, p.col0 + n);
        } else {
          cs.leftv[r] = (p.lcol_in != nullptr && cs.rvalid[r])
                            ? __ldcg(static_cast<const T*>(p.lcol_in) + i)
                            : F::left(p, i);
          cs.rightv[r] = F::right(p, i);
        }
#pragma unroll
        for (int d = 0; d < WV::HV; ++d) cs.hist[r][d] = T(0);
#pragma unroll
        for (int d = 0; d < WV::HC; ++d) cs.hcc[r][d] = CC(0);
      }
#pragma unroll
      for (int d = 0; d < WV::FV; ++d) cs.fifo[d] = T(0);
      const bool virt = strip_top < 0;
      const int K = NQ + D;
      if constexpr (WaveCompute<F, R, SIG, E, W, TABLE, GS>::kVec) {   // staging prologue
        cs.stage_load(p, lane, WV::TAU0);
        cs.stage_load(p, lane, WV::TAU0 + C);
      }
      for (int k = 0; k < K; ++k) {
        const bool has_top = k < NQ;
        const bool has_bot = k >= D;
        const uint32_t gt = iter * (uint32_t)NQ + (uint32_t)k;
        const uint32_t gb = iter * (uint32_t)NQ + (uint32_t)(k - D);
        const T* top = sm.link[wid][0];
        T* bot = sm.link[wid + 1][0];
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
        if (lane == 0) trace_stamp(p, s, wid, W + 2, k, 0);
        const int tau_k = WV::TAU0 + k * C;
        // max column < n-1 keeps the last_col / rcol cells in the checked path
        const bool steady = (tau_k - 31 * D - ((R - 1) / GS) * SIG >= 0) && (tau_k + C < n);
        if (steady && !virt)
          cs.template chunk<0>(p, lane, tau_k, top, bot, has_bot);
        else if (steady)
          cs.template chunk<1>(p, lane, tau_k, top, bot, has_bot);
        else
          cs.template chunk<2>(p, lane, tau_k, top, bot, has_bot);
        __syncwarp();
        if (lane == 0) {
          if (has_top) mbar_arrive(&sm.empty[wid][gt % NS]);
          if (has_bot) mbar_arrive(&sm.full[wid + 1][gb % NS]);
          trace_stamp(p, s, wid, W + 2, k, 1);
        }
      }
      if constexpr (WaveCompute<F, R, SIG, E, W, TABLE, GS>::kVec) {
        cp_async_wait_group<0>();   // staging copies issued past the strip's end must land before the
        __syncwarp();               // next strip's prologue reuses their slots
      }
      // right column of every row of the strip: last_col output and/or rank g+1's window
#pragma unroll
      for (int r = 0; r < R; ++r) {
        if (cs.rvalid[r]) {
          if (p.last_col != nullptr) static_cast<T*>(p.last_col)[cs.irow[r]] = cs.rlast[r];
          if (p.rcol_out != nullptr) static_cast<T*>(p.rcol_out)[cs.irow[r]] = cs.rlast[r];
        }
      }
      if (p.rcol_out != nullptr) __threadfence_system();
    } else if (wid == W) {
      // ------------------------------------------------------------------ loader warp
      // Moves up to kBatch chunks per round trip: one flag check covers every chunk the
      // previous strip has already published, and all their loads are in flight together.
      const T* prev = static_cast<const T*>(p.bnd) + (int64_t)(s - 1) * p.bnd_stride;
      uint64_t avail = 0;   // chunks of strip s-1 known to be published
      int k = 0;
      while (k < NQ) {
        int nb = min(kBatch, NQ - k);
        if (s > 0) {
          if ((uint64_t)(k + 1) > avail) {
            uint64_t seen;
            if (!wait_flag_relaxed(p.prog + (s - 1), ep | (uint64_t)(k + 1), ctl, tmo, seen)) return;
            avail = seen - ep;
          }
          nb = min(nb, (int)(avail - (uint64_t)k));
        }
        if (lane == 0) trace_stamp(p, s, wid, W + 2, k, 0);
        T v[kBatch];
        CC cc[kBatch];
#pragma unroll
        for (int j = 0; j < kBatch; ++j) {
          const int q = (k + j) * C + lane;
          const int c = q - 32;
          if (j < nb) {
            v[j] = (s > 0) ? __ldcg(prev + q) : F::top(p, c + p.col0);
            cc[j] = (c >= 0 && c < n) ? F::col_ctx(p, c + p.col0) : CC(0);
          }
        }
#pragma unroll
        for (int j = 0; j < kBatch; ++j) {
          if (j < nb) {
            const uint32_t g = iter * (uint32_t)NQ + (uint32_t)(k + j);
            const int slot = g % NS;
            if (g / NS >= 1) {
              if (!mbar_wait(&sm.empty[0][slot], ((g / NS) - 1) & 1u, ctl, tmo)) return;
            }
            sm.link[0][slot][lane] = v[j];
            if (!F::kGridIn) sm.bring[((k + j) * C + lane) & (kBRing - 1)] = cc[j];
            __syncwarp();
            if (lane == 0) mbar_arrive(&sm.full[0][slot]);
          }
        }
        if (lane == 0) trace_stamp(p, s, wid, W + 2, k, 1);
        k += nb;
      }
    } else {
      // ------------------------------------------------------------------ storer warp
      // Drains every chunk warp W-1 has already completed (up to kBatch) per round trip and
      // publishes them with one release of the strip's progress flag.
      const bool last = (s == p.nstrips - 1);
      T* mine = static_cast<T*>(p.bnd) + (int64_t)s * p.bnd_stride;
      T rmin = T(0);
      bool have = false;
      int k = 0;
      while (k < NQ) {
        const uint32_t g0 = iter * (uint32_t)NQ + (uint32_t)k;
        if (!mbar_wait(&sm.full[W][g0 % NS], (g0 / NS) & 1u, ctl, tmo)) return;
        int nb = 1;
        if (lane == 0) {
          while (nb < kBatch && k + nb < NQ) {
            const uint32_t g = g0 + (uint32_t)nb;
            if (!mbar_try_wait(&sm.full[W][g % NS], (g / NS) & 1u)) break;
            ++nb;
          }
        }
        nb = __shfl_sync(0xffffffffu, nb, 0);
        if (lane == 0) trace_stamp(p, s, wid, W + 2, k, 0);
        T v[kBatch];
#pragma unroll
        for (int j = 0; j < kBatch; ++j) {
          if (j < nb) {
            const uint32_t g = g0 + (uint32_t)j;
            if (j > 0) mbar_wait(&sm.full[W][g % NS], (g / NS) & 1u, ctl, tmo);   // already complete
            v[j] = sm.link[W][g % NS][lane];
          }
        }
        __syncwarp();
        if (lane == 0) {
#pragma unroll
          for (int j = 0; j < kBatch; ++j)
            if (j < nb) mbar_arrive(&sm.empty[W][(g0 + (uint32_t)j) % NS]);
        }
#pragma unroll
        for (int j = 0; j < kBatch; ++j) {
          if (j < nb) {
            const int q = (k + j) * C + lane;
            const int c = q - 32;
            if (!last) {
              __stcg(mine + q, v[j]);
            } else if (c >= 0 && c < n) {
              if (p.last_row != nullptr) static_cast<T*>(p.last_row)[c] = v[j];
              if (F::kScore == SCORE_LAST_CELL && c == n - 1 && p.score != nullptr && p.is_last_rank)
                *static_cast<T*>(p.score) = v[j];
              if (F::kScore == SCORE_ROW_MIN) {
                rmin = have ? min(rmin, v[j]) : v[j];
                have = true;
              }
            }
          }
        }
        if (!last) {
          __syncwarp();   // orders every lane's stores before lane 0's (cumulative) release
          if (lane == 0) st_release_gpu(p.prog + s, ep | (uint64_t)(k + nb));
        }
        if (lane == 0) trace_stamp(p, s, wid, W + 2, k, 1);
        k += nb;
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
