// adiag.cuh -- lane-systolic persistent kernel for the Anti-Diagonal category (t = i + j,
// Fig. 2 [L117-L122]; §III.A [L148-L168]) with contributing set {L, UL, U} (Table I row
// "Y Y Y N" [L139]): LCS, Levenshtein and DTW.  One launch per fill (no launch per diagonal,
// the paper's K1 [L150]).
//
// Decomposition:
//  * STRIPS of SH = W*32*R rows, bottom-aligned so the last strip ends at row m-1.  Rows above
//    row 0 in strip 0 are VIRTUAL: they carry f-specific constants (F::vrow / F::vbig) chosen so
//    that f itself regenerates the top initialisation in row -1 -- strip 0 runs the same
//    select-free code as every other strip (the first strip paces the whole pipeline).
//  * A CTA of W warps claims strips in increasing order (atomic counter): a strip waits only on
//    the strip above, claimed earlier by a running CTA, so no co-residency is assumed.
//  * Warp w owns rows [top_w, top_w + 32R); lane k owns R consecutive rows and at step tau
//    processes column c = tau - k*E.  The R rows of a lane are chained inside a step (row r's U
//    is row r-1's new value); row 0's U arrives from lane k-1 through ONE rotate-by-one
//    __shfl_sync per step (E steps of slack hide its latency); lane 31 injects the warp's top
//    row in that same shuffle, lane 0 receives it.
//  * Handoffs carry (value, tag) 64-bit pairs that are single-copy atomic, so consumers poll the
//    data itself: no flags, no release fences, no loader / storer warps.
//      - warp w -> warp w+1 (same CTA): shared-memory ring of kAdRing chunks of 32 pairs, tag =
//        per-CTA chunk sequence number; back-pressure through a per-warp consumed counter;
//      - last warp of strip s -> first warp of strip s+1: strip s's boundary row in global
//        memory (L2), tag = the fill's epoch (written once per fill, no back-pressure needed).
//    Consumers validate per group of 8 steps, so a warp lags the warp above by 32E + 8 steps.
//  * The DP table is virtual: only boundary rows (L2-resident) and requested outputs touch
//    global memory.
#pragma once
#include <cstdint>
#include <climits>
#include <cstring>
#include "cellfn.cuh"
#include "params.h"
#include "sync.cuh"

namespace lddp {

// 8-step groups per loop iteration (measured on B200: LCS / Levenshtein 2, DTW 4 -- C5 8.36 ->
// 7.86 ms, C2 1.13 -> 1.00 ms against 1; LDDP_AD_GUNROLL overrides for experiments)
// group of a chunk at which the next chunk's strip-boundary pairs are loaded (kAdHalfPf); measured
// on B200: LCS C5 6.27 / 6.12 / 5.80 ms at group 2 / 1 / 0 -- an early load hides the L2 latency
// better than a stale pair costs
#ifndef LDDP_AD_PG_MATCH
#define LDDP_AD_PG_MATCH 0
#endif
#ifndef LDDP_AD_PG_OTHER
#define LDDP_AD_PG_OTHER 2
#endif
template <class F> constexpr int kAdPfGroup = F::kMatchCells ? LDDP_AD_PG_MATCH : LDDP_AD_PG_OTHER;
#ifdef LDDP_AD_GUNROLL
template <class F> constexpr int kAdGroupUnroll = LDDP_AD_GUNROLL;
#else
template <class F> constexpr int kAdGroupUnroll = F::kMatchCells ? 2 : 4;
#endif
constexpr int kAdRing = 8;   // chunks (of 32 entries) per intra-CTA ring
constexpr int kAdCRing = 256;  // per-warp column-context ring (entries), index = column & 255,
                               // plus an 8-entry overhang mirroring slots 0..7 (no wrap per step)

__device__ __forceinline__ uint64_t ad_ld_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
// the same load for prefetches whose staleness the tag check catches: no memory clobber, so the
// scheduler may still move other memory operations around it (volatile: never speculated out of
// its predicate -- a non-volatile asm was hoisted past the bounds check)
__device__ __forceinline__ uint64_t ad_ld_gpu_pf(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ void ad_st_gpu2(uint64_t* p, uint64_t a, uint64_t b) {
  asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ uint64_t ad_ld_smem(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.volatile.shared.u64 %0, [%1];" : "=l"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void ad_st_smem2(uint64_t* p, uint64_t a, uint64_t b) {
  asm volatile("st.volatile.shared.v2.u64 [%0], {%1, %2};" ::"r"(smem_u32(p)), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ int ad_ld_smem_i32(const int* p) {
  int v;
  asm volatile("ld.volatile.shared.s32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void ad_st_smem_i32(int* p, int v) {
  asm volatile("st.volatile.shared.s32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}

template <class T>
__device__ __forceinline__ uint32_t ad_bits(T v) {
  uint32_t x;
  memcpy(&x, &v, 4);
  return x;
}
template <class T>
__device__ __forceinline__ T ad_val(uint64_t pr) {
  const uint32_t x = (uint32_t)pr;
  T v;
  memcpy(&v, &x, 4);
  return v;
}
__device__ __forceinline__ uint64_t ad_pair(uint32_t bits, uint32_t tag) {
  return ((uint64_t)tag << 32) | bits;
}

// S = 1 ("split"): the lane's rows [R/2, R) run one column behind rows [0, R/2) -- their U at
// column c-1 is the upper half's value from the previous step -- so a step holds two independent
// chains of R/2 cells (ILP 2) for one extra step of lane lag (ELAG = E + S).
template <class F, int R, int W, int E, int S = 0, bool TB = false>
struct AdWarp {
  // TB: TABLE output -- every cell of the strip goes to the row-major table.  A lane's R values
  // per step are staged in a per-warp shared tile [R][32 lanes][33] (conflict-free both ways); at
  // the end of each chunk the warp writes the tile row by row, 32 consecutive columns per store
  // (coalesced), skipping virtual rows and columns outside [0, n).
  static_assert(!TB || !S, "TABLE output: unsplit geometries");
  static constexpr int ELAG = E + S;   // lane-to-lane column lag
  // strip-boundary pairs loaded half a chunk ahead inside the group loop: DTW (fully unrolled
  // groups) and one-warp CTAs (every warp reads its top row from global memory); for 4-warp
  // LCS CTAs the load inside the 2-group loop cost every warp more than it saved warp 0
  static constexpr bool kAdHalfPf = kAdGroupUnroll<F> == 4 || W == 1;
  static constexpr int H2 = S ? R / 2 : R;
  static_assert(!S || (R % 2 == 0), "split needs an even R");
  using T = typename F::T;
  using RC = typename F::RowCtx;
  using CC = typename F::ColCtx;
  static_assert(sizeof(T) == 4, "32-bit cells");
  static_assert(!F::kMatchCells || R <= 8, "match-table entries are 8-bit row masks");
  static constexpr int SH = W * 32 * R;

  // ---- per-lane state
  T hist[R];        // row r's value at the previous step (L of this step)
  T fifo[E + 1];    // fifo[d] = value received from lane k-1 at the end of step tau-1-d
  RC rc[R];         // row contexts (a_i / x_i, or F::vrow() for virtual rows)
  T leftv[R];       // column -1 of each row
  T rlast[R];       // column n-1 of each row (captured in checked chunks)
  CC ccur[8];       // column contexts of the current 8-step group
  CC cprv;          // split: context of the lower half's column (the previous step's)
  T midUL;          // split: upper half's last row two steps back (UL of the lower half)
  CC cpend;         // column context of column 32(k+2) + lane, staged into the ring at chunk k+1
  CC* cring;        // this warp's column-context ring (shared memory)
  uint8_t* mtab;    // match cells: this warp's table mtab[c * 32 + lane] = rows r of the lane with
                    // a_r == c (bit r), c in [0, 256) (dynamic shared memory)
  uint8_t* ctab;    // match cells, small alphabets: this warp's code table, byte c -> code 0..3 of
                    // the warp's <= 4 distinct row characters, 4 for any other byte
  uint32_t mpk;     // ... and this lane's masks packed by code (byte k = rows with code k)
  uint32_t* cnib;   // small alphabets: the warp's column codes, 4 bits per column, 8 per word
                    // (32 words for the 256-column ring + 1 mirrored word for the funnel read)
  bool small;       // warp-uniform: the warp's rows use <= 4 distinct characters -> the column
                    // ring holds codes and a step's mask is one PRMT of mpk (no table lookup)
  int32_t one;      // run-time 1 held in a register (opaque to ptxas: no per-use constant loads)
  int64_t irow0;    // global row of this lane's row 0
  uint32_t* tbl;    // TB: this warp's staging tile (32 * R * 33 words)

  // ---- per-warp handoff state
  uint64_t tp;      // this lane's top pair of the current chunk (column 32k + lane)
  uint64_t tq1;     // global top prefetch (chunk k+1)
  const uint64_t* tqsrc;   // TS 2: this lane's slot of the previous strip's boundary row (column
                           // 32k + lane at tqsrc + 32k); the next chunk's pair is loaded inside the
                           // group loop at group kAdPfGroup (0 for LCS / Levenshtein, 2 for DTW)
  int tqn;                 // chunks with a global top pair (NQ), 0 for other roles
  long long wait_top; // clock64 cycles spent waiting for top values (trace builds)

  __device__ __forceinline__ CC colctx_guard(const FillParams& p, int c) const {
    return ((unsigned)c < (unsigned)p.cols) ? F::col_ctx(p, c + p.col0) : CC(0);
  }
  __device__ __forceinline__ T leftval(const FillParams& p, int64_t i) const {
    if (i >= 0) {
      if (p.lcol_in != nullptr) return __ldcg(static_cast<const T*>(p.lcol_in) + i);
      return F::left(p, i);
    }
    if (i == -1) return F::top(p, p.col0 - 1);
    return F::vbig();
  }

  // Shared-memory / global handoff endpoints of this warp for one strip.
  struct Links {
    uint64_t* ring_top;        // ring[w][0][0]     (TS 1)
    uint64_t* ring_bot;        // ring[w + 1][0][0] (BS 1)
    int* cons_self;            // &cons[w]          (TS 1)
    const int* cons_next;      // &cons[w + 1]      (BS 1)
    const uint64_t* gprev;     // strip s-1's boundary row (TS 2)
    uint64_t* gmine;           // strip s's boundary row   (BS 2)
    T* stg;                    // this warp's bottom staging row (32 values, shared memory)
    T* tstg;                   // this warp's top staging row: chunk k's 32 top values
    uint32_t base;             // ring chunk tag of chunk 0 in this strip
    uint32_t ep32;             // epoch tag of the global boundary pairs
    bool top_init;             // TS 0: the row above is table row 0 (else a virtual row)
    long long wait_bp;
  };

  // ------------------------------------------------------------------ chunk-level handoffs
  // Top pairs of chunk k (columns 32k + lane): all 32 validated before the chunk's steps run.
  __device__ __forceinline__ bool acquire_top(const FillParams& p, const int lane, const int k, const int NQ,
                                              const int TS, Links& lk, Control* ctl) {
    if (k >= NQ) return true;   // columns >= n: the injected values are never used
    if (TS == 0) {
      const T v = lk.top_init ? F::top(p, 32 * k + lane + p.col0) : F::vbig();
      tp = ad_pair(ad_bits(v), 0u);
      return true;
    }
    const uint64_t* src;
    uint32_t tag;
    if (TS == 1) {
      src = lk.ring_top + (k % kAdRing) * 32 + lane;
      tag = lk.base + (uint32_t)k;
      tp = ad_ld_smem(src);
    } else {
      src = lk.gprev + 32 * (int64_t)k + lane;
      tag = lk.ep32;
      tp = tq1;
      // next chunk's pair: half a chunk ahead inside the group loop (kAdHalfPf), else here
      if constexpr (!kAdHalfPf) tq1 = (k + 1 < NQ) ? ad_ld_gpu(src + 32) : 0ull;
    }
    if (__all_sync(0xffffffffu, (uint32_t)(tp >> 32) == tag)) return true;
    const long long t0 = clock64();
    Backoff w;
    int spins = 0;
    while (true) {
      if ((uint32_t)(tp >> 32) != tag) tp = (TS == 1) ? ad_ld_smem(src) : ad_ld_gpu(src);
      if (__all_sync(0xffffffffu, (uint32_t)(tp >> 32) == tag)) break;
      // busy-poll first (a mid-strip wait is normally one hop of latency: sleeping there adds to
      // the pipeline lag of every warp below), then back off
      if (++spins > p.spin_polls && !w.tick(ctl, p.timeout_ns)) return false;
    }
    wait_top += clock64() - t0;
    return true;
  }

  // Bottom chunk j (columns 32j + lane), staged by lane 31 in lk.stg during the chunk that
  // produced it, published as tagged pairs (ring / global) or plain last-row values.
  __device__ __forceinline__ bool publish_bottom(const FillParams& p, const int lane, const int j, const int NQ,
                                                 const int BS, Links& lk, Control* ctl) {
    if (BS == 0 || j < 0 || j >= NQ) return true;
    __syncwarp();
    const T v = lk.stg[lane];
    __syncwarp();
    if (BS == 1) {
      const uint32_t tag = lk.base + (uint32_t)j;
      if (j >= kAdRing) {   // warp w+1 must have consumed chunk j - kAdRing (same ring slot)
        if ((int)((uint32_t)ad_ld_smem_i32(lk.cons_next) - (tag - kAdRing)) < 0) {
          const long long t0 = clock64();
          Backoff w;
          while ((int)((uint32_t)ad_ld_smem_i32(lk.cons_next) - (tag - kAdRing)) < 0)
            if (!w.tick(ctl, p.timeout_ns)) return false;
          lk.wait_bp += clock64() - t0;
        }
      }
      uint64_t* d = lk.ring_bot + (j & (kAdRing - 1)) * 32 + lane;
      asm volatile("st.volatile.shared.u64 [%0], %1;" ::"r"(smem_u32(d)), "l"(ad_pair(ad_bits(v), tag)) : "memory");
    } else if (BS == 2) {
      uint64_t* d = lk.gmine + 32 * (int64_t)j + lane;
      asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(d), "l"(ad_pair(ad_bits(v), lk.ep32)) : "memory");
    } else {
      const int c = 32 * j + lane;
      if (c < p.cols) static_cast<T*>(p.last_row)[c] = v;
    }
    return true;
  }

  // One chunk = 32 steps tau = 32k - E + su, su = 0..31, in 4 groups of 8.
  //  top: lane su's tp holds the top value of column 32k + su, injected by lane 31 at step su
  //  bottom: lane 31's row R-1 at step su is column 32(k - E) + su of the warp's bottom row;
  //          it is staged in shared memory (two STS.128 per group) and published next chunk
  // CHECKED: boundary columns -1 / n-1 (left values, right-column capture).
  // The 8-step body is identical for every warp role (no role branches inside it), so ptxas
  // can overlap consecutive steps and the body stays small for the instruction cache.
  template <bool CHECKED, bool SM>
  __device__ __forceinline__ void chunk(const FillParams& p, const int lane, const int k, T* stg, T* tstg) {
    const int n = p.cols;
    const int lane_off = lane * ELAG;
    const T topv = ad_val<T>(tp);
    // column contexts: one coalesced load per 32 columns, two chunks ahead, staged through the
    // warp's shared ring (the body reads it with LDS: lower latency than L1 hits)
    {
      const int slot = (32 * (k + 1) + lane) & (kAdCRing - 1);
      if constexpr (F::kMatchCells && SM) {
        // 8 lanes' codes -> one word of nibbles (column slot 8w + j at bits 4j)
        uint32_t v = (uint32_t)ctab[(uint32_t)cpend & 255u] << (4 * (lane & 7));
        v |= __shfl_xor_sync(0xffffffffu, v, 1);
        v |= __shfl_xor_sync(0xffffffffu, v, 2);
        v |= __shfl_xor_sync(0xffffffffu, v, 4);
        if ((lane & 7) == 0) {
          cnib[slot >> 3] = v;
          if (slot == 0) cnib[kAdCRing / 8] = v;
        }
      } else {
        cring[slot] = cpend;
        if (slot < 8) cring[slot + kAdCRing] = cpend;
      }
    }
    cpend = colctx_guard(p, 32 * (k + 2) + lane);
    // chunk k's top row -> shared memory; lane 31 takes its 8 injections per group from there,
    // loaded one group ahead (off the rotate-SHFL chain)
    __syncwarp();
    tstg[lane] = topv;
    __syncwarp();
    T injq[8];
    {
      const uint4 i0 = reinterpret_cast<const uint4*>(tstg)[0];
      const uint4 i1 = reinterpret_cast<const uint4*>(tstg)[1];
      injq[0] = ad_val<T>(i0.x); injq[1] = ad_val<T>(i0.y); injq[2] = ad_val<T>(i0.z); injq[3] = ad_val<T>(i0.w);
      injq[4] = ad_val<T>(i1.x); injq[5] = ad_val<T>(i1.y); injq[6] = ad_val<T>(i1.z); injq[7] = ad_val<T>(i1.w);
    }
#pragma unroll(kAdGroupUnroll<F>)
    for (int g = 0; g < 4; ++g) {
      // a relaxed gpu-scope L2 load (in the memory model: it races the producer's relaxed pair
      // store; predicated, no branch in the group body); a stale pair is caught by the tag check
      // and re-polled in acquire_top
      if constexpr (kAdHalfPf) {
        if (g == kAdPfGroup<F> && k + 1 < tqn) tq1 = ad_ld_gpu_pf(reinterpret_cast<const uint64_t*>(tqsrc) + 32 * (k + 1));
      }
      CC cnext[8];
      const int tau0 = 32 * k - E + 8 * g;
      if constexpr (F::kMatchCells && SM) {
        // the next group's 8 column codes (one funnel shift of two words), then two PRMTs give
        // the 8 steps' match masks (code 4 selects a zero byte: matches nothing)
        const int cn = (tau0 + 8 - lane_off) & (kAdCRing - 1);
        const uint32_t codes = __funnelshift_r(cnib[cn >> 3], cnib[(cn >> 3) + 1], 4 * (cn & 7));
        const uint32_t m0 = __byte_perm(mpk, 0u, codes);
        const uint32_t m1 = __byte_perm(mpk, 0u, codes >> 16);
#pragma unroll
        for (int u = 0; u < 8; ++u) cnext[u] = CC((u < 4 ? m0 : m1) >> (8 * (u & 3)));
      } else {
        const CC* cr = cring + ((tau0 + 8 - lane_off) & (kAdCRing - 1));
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          if constexpr (F::kMatchCells) cnext[u] = CC(mtab[(uint32_t)cr[u] * 32 + lane]);
          else cnext[u] = cr[u];
        }
      }
      T injn[8];
      if (g < 3) {
        const uint4 i0 = reinterpret_cast<const uint4*>(tstg + 8 * g + 8)[0];
        const uint4 i1 = reinterpret_cast<const uint4*>(tstg + 8 * g + 8)[1];
        injn[0] = ad_val<T>(i0.x); injn[1] = ad_val<T>(i0.y); injn[2] = ad_val<T>(i0.z); injn[3] = ad_val<T>(i0.w);
        injn[4] = ad_val<T>(i1.x); injn[5] = ad_val<T>(i1.y); injn[6] = ad_val<T>(i1.z); injn[7] = ad_val<T>(i1.w);
      }
      T bv[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = tau0 + u - lane_off;
        const CC cc = ccur[u];
        T U = fifo[E - 1];
        T UL = fifo[E];
        T nw[R];
        if constexpr (S) {
          // upper half at column c, lower half at column c-1: two independent chains, interleaved
          const int cl = c - 1;
          T UB = hist[H2 - 1];   // upper row H2-1 at column c-1 (previous step)
          T ULB = midUL;         // ... at column c-2
#pragma unroll
          for (int r = 0; r < H2; ++r) {
            T v, w;
            const int q = H2 + r;
            if constexpr (F::kMatchCells) {
              v = F::fadm(hist[r], UL, U, ((uint32_t)cc >> r) & 1u, one);
              w = F::fadm(hist[q], ULB, UB, ((uint32_t)cprv >> q) & 1u, one);
            } else {
              v = F::fad(hist[r], UL, U, rc[r], cc, one);
              w = F::fad(hist[q], ULB, UB, rc[q], cprv, one);
            }
            if (CHECKED) {
              v = (c == -1) ? leftv[r] : v;
              rlast[r] = (c == n - 1) ? v : rlast[r];
              w = (cl == -1) ? leftv[q] : w;
              rlast[q] = (cl == n - 1) ? w : rlast[q];
            }
            UL = hist[r];
            U = v;
            nw[r] = v;
            ULB = hist[q];
            UB = w;
            nw[q] = w;
          }
          midUL = hist[H2 - 1];
          cprv = cc;
        } else {
#pragma unroll
          for (int r = 0; r < R; ++r) {
            T v;
            if constexpr (F::kMatchCells) v = F::fadm(hist[r], UL, U, ((uint32_t)cc >> r) & 1u, one);
            else v = F::fad(hist[r], UL, U, rc[r], cc, one);
            if (CHECKED) {
              v = (c == -1) ? leftv[r] : v;
              rlast[r] = (c == n - 1) ? v : rlast[r];
            }
            UL = hist[r];
            U = v;
            nw[r] = v;
            if constexpr (TB) tbl[(r * 32 + lane) * 33 + 8 * g + u] = ad_bits(v);
          }
        }
        bv[u] = nw[R - 1];
        const T inj = injq[u];
        const T sv = (lane == 31) ? inj : nw[R - 1];
        const T rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
        for (int d = E; d > 0; --d) fifo[d] = fifo[d - 1];
        fifo[0] = rv;
#pragma unroll
        for (int r = 0; r < R; ++r) hist[r] = nw[r];
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        ccur[u] = cnext[u];
        if (g < 3) injq[u] = injn[u];
      }
      if (lane == 31) {
        uint4* d = reinterpret_cast<uint4*>(stg + 8 * g);
        d[0] = make_uint4(ad_bits(bv[0]), ad_bits(bv[1]), ad_bits(bv[2]), ad_bits(bv[3]));
        d[1] = make_uint4(ad_bits(bv[4]), ad_bits(bv[5]), ad_bits(bv[6]), ad_bits(bv[7]));
      }
    }
    if constexpr (TB) store_tile(p, lane, k);
  }

  // TB: the chunk's tile -> table.  Row r of lane src holds columns 32k - E - src * ELAG + su at
  // tile [(r * 32 + src) * 33 + su]; lane su of the warp stores that column (one coalesced row
  // segment per (src, r)).
  __device__ __forceinline__ void store_tile(const FillParams& p, const int lane, const int k) {
    __syncwarp();
    const int n = p.cols;
    const int64_t m = p.rows;
    const int64_t wtop = irow0 - (int64_t)lane * R;
    const int64_t pitch = p.table_pitch;
    // this lane's column for src = 0 and the pointer of (src = 0, r = 0); src + 1 is R rows down
    // and ELAG columns left
    const int col0 = 32 * k - E + lane;
    uint32_t* rowp = static_cast<uint32_t*>(p.table) + wtop * pitch + col0;
    const int64_t step_src = (int64_t)R * pitch - ELAG;
    const bool fast = (32 * k - E - 31 * ELAG >= 0) && (32 * k - E + 31 < n) && wtop >= 0 && wtop + 32 * R <= m;
    if (__all_sync(0xffffffffu, fast)) {   // every (row, column) of the tile inside the table
#pragma unroll 4
      for (int src = 0; src < 32; ++src) {
#pragma unroll
        for (int r = 0; r < R; ++r) rowp[r * pitch] = tbl[(r * 32 + src) * 33 + lane];
        rowp += step_src;
      }
    } else {
#pragma unroll 4
      for (int src = 0; src < 32; ++src) {
        const int col = col0 - src * ELAG;
        const bool cin = (unsigned)col < (unsigned)n;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int64_t row = wtop + (int64_t)src * R + r;
          const uint32_t v = tbl[(r * 32 + src) * 33 + lane];
          if (cin && row >= 0 && row < m) rowp[r * pitch] = v;
        }
        rowp += step_src;
      }
    }
    __syncwarp();
  }

  template <bool CHECKED, bool SM>
  __device__ __forceinline__ bool step_chunk(const FillParams& p, const int lane, const int k, const int NQ,
                                             const int TS, const int BS, Links& lk, Control* ctl) {
    // the staging row holds bottom chunk k-1-E (produced during chunk k-1): publish it first
    if (!publish_bottom(p, lane, k - 1 - ELAG, NQ, BS, lk, ctl)) return false;
    if (!acquire_top(p, lane, k, NQ, TS, lk, ctl)) return false;
    // ring chunk k is in registers now: release its slot to warp w-1
    if (TS == 1 && k < NQ && lane == 0) ad_st_smem_i32(lk.cons_self, (int)(lk.base + (uint32_t)k));
    chunk<CHECKED, SM>(p, lane, k, lk.stg, lk.tstg);
    return true;
  }

  // All K = NQ + E chunks of one strip: checked chunks at both ends, a tight steady loop between.
  // TS / BS are warp-uniform run-time roles handled at chunk granularity only.
  template <bool SM>
  __device__ __forceinline__ bool strip(const FillParams& p, const int lane, const int NQ, const int TS,
                                        const int BS, Links& lk, Control* ctl) {
    const int n = p.cols;
    const int K = NQ + ELAG;
    const int k0 = min(ELAG, K);
    // steady: every lane's columns in [0, n-1) (no boundary column in the chunk)
    int k1 = (n - 33 + E) >= 0 ? (n - 33 + E) / 32 + 1 : 0;
    k1 = max(k0, min(K, k1));
    for (int k = 0; k < k0; ++k)
      if (!step_chunk<true, SM>(p, lane, k, NQ, TS, BS, lk, ctl)) return false;
    for (int k = k0; k < k1; ++k)
      if (!step_chunk<false, SM>(p, lane, k, NQ, TS, BS, lk, ctl)) return false;
    for (int k = k1; k < K; ++k)
      if (!step_chunk<true, SM>(p, lane, k, NQ, TS, BS, lk, ctl)) return false;
    return publish_bottom(p, lane, K - 1 - ELAG, NQ, BS, lk, ctl);   // the last staged chunk
  }
};

template <class F, int R, int W, int E, int S = 0, bool TB = false>
__global__ void __launch_bounds__(W * 32, 1) adiag_kernel(const FillParams p) {
  using AW = AdWarp<F, R, W, E, S, TB>;
  static_assert(!TB || W == 1, "TABLE output: one-warp strips");
  static_assert(!TB || sizeof(typename F::OutT) == 4, "TABLE output: 32-bit cells");
  __shared__ uint32_t tbl_sh[TB ? W : 1][TB ? 32 * R * 33 : 1];   // TB staging tiles
  using T = typename AW::T;
  constexpr int SH = AW::SH;
  __shared__ __align__(16) uint64_t ring[W][kAdRing][32];   // ring[w]: top stream of warp w >= 1
  __shared__ int cons[W];                                   // last chunk tag consumed by warp w
  __shared__ typename F::ColCtx cring[W][kAdCRing + 8];    // per-warp column-context rings
  __shared__ __align__(16) T stg[W][32];                   // per-warp bottom staging row
  __shared__ __align__(16) T tstg[W][32];                  // per-warp top staging row
  __shared__ int strip_sh;
  __shared__ int one_sh;
  extern __shared__ __align__(16) uint8_t ad_dyn_smem[];    // match tables (W x 256 x 32 u8)
  __shared__ uint8_t ctab_sh[W][256];                       // per-warp small-alphabet code tables
  __shared__ uint32_t cnib_sh[W][kAdCRing / 8 + 1];         // per-warp column codes (nibbles)

  Control* ctl = static_cast<Control*>(p.ctl);
  const int lane = threadIdx.x & 31;
  const int wid = threadIdx.x >> 5;
  const int n = p.cols;
  const int NQ = (n + 31) / 32;   // top / bottom chunks per strip

  const uint32_t ep32 = (uint32_t)p.epoch;

  for (int i = threadIdx.x; i < W * kAdRing * 32; i += blockDim.x) (&ring[0][0][0])[i] = 0ull;
  if (threadIdx.x < W) cons[threadIdx.x] = 0;
  if (threadIdx.x == 0) one_sh = p.one;
  __syncthreads();

  uint32_t iter = 0;
  while (true) {
    if (threadIdx.x == 0) {
      int s = (int)atomicAdd(&ctl->claim, 1u);
      if (ld_volatile_u32(&ctl->abort)) s = INT_MAX;
      strip_sh = s;
    }
    __syncthreads();
    const int s = strip_sh;
    if (s >= p.nstrips) break;
    const int64_t strip_top = p.row0 + (int64_t)s * SH;
    const int64_t wtop = strip_top + (int64_t)wid * 32 * R;
    const bool last_strip = (s == p.nstrips - 1);
    const uint32_t base = iter * (uint32_t)NQ + 1u;   // ring chunk tags of this strip

    AW aw;
    bool ok = true;
    // multi-GPU: rank g-1's right column of this strip and the previous strip's last row
    if (p.lcol_in != nullptr) ok = window_consume_wait(p, s, ctl);
    aw.irow0 = wtop + (int64_t)lane * R;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t i = aw.irow0 + r;
      aw.rc[r] = (i >= 0) ? F::row_ctx(p, i) : F::vrow();
      aw.leftv[r] = aw.leftval(p, i);
      aw.rlast[r] = T(0);
      aw.hist[r] = T(0);
    }
    aw.midUL = T(0);
    aw.cprv = typename F::ColCtx(0);
#pragma unroll
    for (int d = 0; d <= E; ++d) aw.fifo[d] = T(0);
    // lane 0's UL at column 0: the row above the warp at column -1 (received "before" step -E)
    if (lane == 0) aw.fifo[0] = aw.leftval(p, wtop - 1);
    if (p.lcol_in != nullptr) {   // every left value of the strip is in registers: release the slot
      __syncthreads();
      if (threadIdx.x == 0 && ok) window_consume_ack(p, s);
    }
    aw.cring = cring[wid];
    aw.tbl = tbl_sh[TB ? wid : 0];
    aw.one = ad_ld_smem_i32(&one_sh);   // a volatile load: ptxas cannot rematerialise it per use
    aw.small = false;
    if constexpr (F::kMatchCells) {
      // Code table of the warp's row characters: if they take <= 4 distinct byte values (DNA),
      // every step's match mask is one PRMT of a per-lane packed register instead of a table load.
      aw.mtab = ad_dyn_smem + wid * 256 * 32;
      aw.ctab = ctab_sh[wid];
#pragma unroll
      for (int j = 0; j < 8; ++j) aw.ctab[8 * lane + j] = 0xFF;
      __syncwarp();
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int c = (int)aw.rc[r];
        if (c >= 0 && c < 256) aw.ctab[c] = 0;   // present (benign same-value races)
      }
      __syncwarp();
      uint32_t pb = 0;
#pragma unroll
      for (int j = 0; j < 8; ++j) pb |= (aw.ctab[8 * lane + j] == 0 ? 1u : 0u) << j;
      const int cnt = __popc(pb);
      int pre = cnt;   // inclusive warp prefix sum of the distinct-character counts
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, pre, off);
        if (lane >= off) pre += t;
      }
      const int total = __shfl_sync(0xffffffffu, pre, 31);
      aw.small = total <= 4;
      __syncwarp();
      if (aw.small) {
        const int base0 = pre - cnt;
#pragma unroll
        for (int j = 0; j < 8; ++j)
          aw.ctab[8 * lane + j] = ((pb >> j) & 1u) ? (uint8_t)(base0 + __popc(pb & ((1u << j) - 1u))) : (uint8_t)4;
        __syncwarp();
        aw.mpk = 0;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int c = (int)aw.rc[r];
          if (c >= 0 && c < 256) aw.mpk |= 1u << (8 * aw.ctab[c] + r);
        }
      } else {
        // this warp's match table for its lanes' rows (virtual rows match nothing)
        for (int c = 0; c < 256; ++c) aw.mtab[c * 32 + lane] = 0;
        __syncwarp();
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int c = (int)aw.rc[r];
          if (c >= 0 && c < 256) aw.mtab[c * 32 + lane] |= (uint8_t)(1u << r);
        }
      }
      __syncwarp();
    }
    aw.cnib = cnib_sh[wid];
    for (int q = -E - 1 - S; q <= 0; ++q) {
      const int slot = (32 * q + lane) & (kAdCRing - 1);
      typename F::ColCtx v = aw.colctx_guard(p, 32 * q + lane);
      if constexpr (F::kMatchCells) {
        if (aw.small) {
          uint32_t w = (uint32_t)aw.ctab[(uint32_t)v & 255u] << (4 * (lane & 7));
          w |= __shfl_xor_sync(0xffffffffu, w, 1);
          w |= __shfl_xor_sync(0xffffffffu, w, 2);
          w |= __shfl_xor_sync(0xffffffffu, w, 4);
          if ((lane & 7) == 0) {
            aw.cnib[slot >> 3] = w;
            if (slot == 0) aw.cnib[kAdCRing / 8] = w;
          }
        }
      }
      aw.cring[slot] = v;
      if (slot < 8) aw.cring[slot + kAdCRing] = v;
    }
    aw.cpend = aw.colctx_guard(p, 32 + lane);
    __syncwarp();
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const typename F::ColCtx c = aw.cring[((-E - lane * AW::ELAG) & (kAdCRing - 1)) + u];
      if constexpr (F::kMatchCells)
        aw.ccur[u] = aw.small ? typename F::ColCtx(__byte_perm(aw.mpk, 0u, (uint32_t)aw.ctab[(uint32_t)c & 255u]))
                              : typename F::ColCtx(aw.mtab[(uint32_t)c * 32 + lane]);
      else aw.ccur[u] = c;
    }

    // top source: 0 = generated (strip 0, warp 0), 1 = smem ring (warp w-1), 2 = global (strip s-1)
    const bool nohand = (p.debug & 1) != 0;   // development: independent warps (wrong results)
    int topsrc = nohand ? 0 : ((wid > 0) ? 1 : (s > 0 ? 2 : 0));
    // bottom sink: 1 = smem ring (warp w+1), 2 = global boundary row, 3 = last_row output
    int botsnk = nohand ? 0 : ((wid < W - 1) ? 1 : (last_strip ? (p.last_row != nullptr ? 3 : 0) : 2));
    if (p.debug & 2) {   // development: no strip-to-strip handoff (wrong results)
      if (topsrc == 2) topsrc = 0;
      if (botsnk == 2) botsnk = 0;
    }
    if (p.debug & 4) {   // development: no warp-to-warp handoff inside the CTA (wrong results)
      if (topsrc == 1) topsrc = 0;
      if (botsnk == 1) botsnk = 0;
    }
    const uint64_t gt0 = globaltimer_ns();
    const long long ck0 = clock64();
    aw.wait_top = 0;
    typename AW::Links lk;
    lk.ring_top = &ring[wid][0][0];
    lk.ring_bot = &ring[(wid + 1) % W][0][0];
    lk.cons_self = &cons[wid];
    lk.cons_next = &cons[(wid + 1) % W];
    lk.gprev = static_cast<const uint64_t*>(p.bnd) + (int64_t)(s - 1) * p.bnd_stride;
    lk.gmine = static_cast<uint64_t*>(p.bnd) + (int64_t)s * p.bnd_stride;
    lk.stg = stg[wid];
    lk.tstg = tstg[wid];
    lk.base = base;
    lk.ep32 = ep32;
    lk.top_init = (strip_top - 1 == -1);
    lk.wait_bp = 0;
    aw.tp = 0;
    aw.tqsrc = lk.gprev + lane;
    aw.tqn = (topsrc == 2) ? NQ : 0;
    if (topsrc == 2) aw.tq1 = ad_ld_gpu(lk.gprev + lane);
    if constexpr (F::kMatchCells)
      ok = ok && (aw.small ? aw.template strip<true>(p, lane, NQ, topsrc, botsnk, lk, ctl)
                           : aw.template strip<false>(p, lane, NQ, topsrc, botsnk, lk, ctl));
    else
      ok = ok && aw.template strip<false>(p, lane, NQ, topsrc, botsnk, lk, ctl);
    const long long wait_bp = lk.wait_bp;
    if (p.trace != nullptr && lane == 0) {   // per (strip, warp): start, end, cycles, waits
      uint64_t* tr = p.trace + ((int64_t)s * W + wid) * 6;
      tr[0] = gt0;
      tr[1] = globaltimer_ns();
      tr[2] = (uint64_t)(clock64() - ck0);
      tr[3] = (uint64_t)aw.wait_top;
      tr[4] = (uint64_t)wait_bp;
      tr[5] = (uint64_t)blockIdx.x;
    }
    // right column of every row: last_col output, rank g+1's window (once rank g+1 has released
    // this slot), the score
    if (p.rcol_out != nullptr) {
      __shared__ int pw_ok;
      __syncthreads();
      if (threadIdx.x == 0) pw_ok = ok && window_produce_wait(p, s, ctl);
      __syncthreads();
      ok = ok && pw_ok;
    }
    if (ok) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int64_t i = aw.irow0 + r;
        if (i >= 0 && i < p.rows) {
          if (p.last_col != nullptr) static_cast<T*>(p.last_col)[i] = aw.rlast[r];
          if (p.rcol_out != nullptr) static_cast<T*>(p.rcol_out)[i] = aw.rlast[r];
          if (i == p.rows - 1 && p.score != nullptr && p.is_last_rank && F::kScore == SCORE_LAST_CELL)
            *static_cast<T*>(p.score) = aw.rlast[r];
        }
      }
      if (p.rcol_out != nullptr) __threadfence_system();
    }
    __syncthreads();
    if (p.rflag_out != nullptr && threadIdx.x == 0 && ok) {
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
