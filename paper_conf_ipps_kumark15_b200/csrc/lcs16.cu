// lcs16.cu -- packed 16x2 lane-systolic kernel for LCS, the anti-diagonal category's default
// for f = LCS (Table I row "Y Y Y N" [L139]; §III.A [L148-L168]; Fig. 1(c) [L88], reading R1).
// One launch per fill, one warp per strip, strips claimed in order.
//
// Why 16x2.  The round-1 adiag body spends ~50 cycles per step on six chained 32-bit cells
// whose match increments are predicated IMADs: the seven predicate registers serialise the
// steps (tools/micro/simd16.cu MODE 0).  Here every register holds TWO cells, so one
// VIMNMX3.U16x2 evaluates max3(U, L, UL + [a_i = b_j]) for two rows, and the match increments
// come from one PRMT per row pair (no predicates): ~21 cycles per step for the same 192 cells
// per warp (MODE 2).
//
// Decomposition: a warp is a 64-lane VIRTUAL warp.
//  * Band A (lo halves): lane k owns rows top + kP + p, p < P.  Band B (hi halves): rows
//    top + 32P + kP + p.  A strip has SH = 64P rows.
//  * At step tau lane k's A rows are at column tau - kE and its B rows at tau - (32 + k)E, so
//    band B is band A's continuation: B's lane 0 takes its top row from A's lane 31 through the
//    same rotate SHFL that carries every lane-to-lane handoff (lane 31 sends (injected top value,
//    own A bottom) packed; a per-lane PRMT selector builds it, no branch).
//  * Match increments: per warp the <= 4 distinct row characters get codes 0..3; per lane and
//    pair p, tabA[p] / tabB[p] hold byte k = [row has code k]; the column ring holds one PRMT
//    selector per column (A's code, B's code, zero bytes between), so
//    m = PRMT(tabA[p], tabB[p], sel) = [a_A = b_cA] + [a_B = b_cB] << 16.
//    Warps whose rows use more than 4 characters take a table path (per-warp match table).
//  * Values are RELATIVE to a warp-uniform base (absolute = relative + base), rebased every 8
//    chunks: every value a warp holds lies within 64P + 64E + 2 of its lane 0 (|LCS(i,j) -
//    LCS(i',j')| <= |i-i'| + |j-j'| over the strip's 64P rows and 64E columns of lane lag), so
//    16 bits hold them (rebase()); all handoffs and outputs are absolute 32-bit.
//  * Boundary columns without per-column selects: before column 0 every lane sweeps "columns"
//    that match nothing, starting from the left boundary values; for LCS max(U, L, UL) there
//    keeps every row at its left value (the left column is non-decreasing downwards), so column
//    -1 arrives by itself.  Past column n-1 the same argument keeps every row at its column n-1
//    value, so the right column is the final register state.  Every chunk runs one body.
//  * Memory traffic in the body: the column characters (cp.async into a per-warp byte ring)
//    and the next chunk's top pairs (cp.async.cg into shared memory) are asynchronous copies:
//    no register scoreboard is left pending across the step loop (a register-destination
//    prefetch shared a scoreboard slot with the loop's LDS / SHFL and stalled it for the L2
//    latency, tools/l16_trace.py).
#include <climits>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "adiag.cuh"

namespace lddp {

namespace l16 {

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t s) {
  uint32_t d;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(s));
  return d;
}
__device__ __forceinline__ uint32_t imad(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}
__device__ __forceinline__ uint32_t pack(int32_t lo, int32_t hi) {
  return ((uint32_t)lo & 0xFFFFu) | ((uint32_t)hi << 16);
}
// PRMT selector nibble of a column code: byte k of the table (k < 4) or a zero byte (byte 0's
// sign replicated: table bytes are 0 / 1)
__device__ __forceinline__ uint32_t selnib(uint32_t code, uint32_t off) { return code < 4 ? off + code : 8u; }
__device__ __forceinline__ void cp_async_cg16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// opaque register copies: ptxas cannot rematerialise them from the constant bank inside the loop
__device__ __forceinline__ int opq(int x) {
  asm volatile("mov.b32 %0, %0;" : "+r"(x));
  return x;
}
template <class T>
__device__ __forceinline__ T* opqp(T* x) {
  asm volatile("mov.b64 %0, %0;" : "+l"(x));
  return x;
}

constexpr int kRing = 256;    // column ring entries (index = column & 255) + 8 mirrored
constexpr int kChr = 1024;    // byte ring of b (index = global byte offset & 1023)
constexpr int kPfGroup = 2;   // group of chunk k at which chunk k+1's top pairs are copied
constexpr int kDynPerWarp = 257 * 32 * 2;   // table path: 257 characters x 32 lanes x u16

}  // namespace l16

// compiled (P row pairs per lane, E lane lag) geometries
#define LDDP_L16_GEOMS \
  LDDP_L16_GEOM(2, 3) LDDP_L16_GEOM(4, 2) LDDP_L16_GEOM(6, 2) LDDP_L16_GEOM(6, 3) LDDP_L16_GEOM(8, 2)

template <int P, int E>
struct L16Warp {
  static constexpr int SH = 64 * P;     // strip rows
  static constexpr int ELAG = 2 * E;    // chunks from a top chunk to the bottom chunk it yields
  static_assert(P >= 1 && P <= 8, "match-table entries hold 8 A rows and 8 B rows");
  static_assert(32 * E + 96 <= l16::kRing, "column ring too small for the band-B lag");

  uint32_t h[P];        // pair p at the previous step (L of this step)
  uint32_t fifo[E];     // fifo[d] = packed value received from lane k-1 at the end of step tau-1-d
  uint32_t U0p;         // U of pair 0 at the previous step (UL of pair 0)
  uint32_t tabA[P], tabB[P];   // small alphabets: byte k = [A / B row p has code k]
  uint32_t ssel;        // sv selector: lane 31 = (injected top lo, own A bottom lo), else identity
  uint32_t one;         // run-time 1 (keeps the +m on the FMA pipe as IMAD)
  int32_t base;         // absolute value = relative + base (warp-uniform)
  uint32_t* ring;       // per-warp column ring (selectors, or packed characters)
  uint8_t* chr;         // per-warp byte ring of b
  const uint8_t* ctab;  // per-warp character -> code table (small path)
  const uint16_t* mtab; // per-warp match table (table path): [c][lane] bits p = A rows, 8+p = B rows;
                        // row 256 stays zero (out-of-range columns)
  uint64_t* pbuf;       // per-warp next-chunk top pairs (cp.async destination)
  const uint8_t* bsrc;  // b (whole string; 4-byte aligned)
  uint64_t tp;          // this lane's top pair of the current chunk (column 32k + lane)
  uint32_t sq[8];       // ring selectors of the current 8-step group (loaded one group ahead)
  long long wait_top;
  uint64_t t_first;     // trace builds: globaltimer after chunk 0's top row was acquired

  // character of local column c, -1 outside [0, n) (matches nothing)
  __device__ __forceinline__ int32_t chr_at(int cols, int col0, int c) const {
    return ((unsigned)c < (unsigned)cols) ? (int32_t)chr[(col0 + c) & (l16::kChr - 1)] : -1;
  }
  template <bool SM>
  __device__ __forceinline__ uint32_t ring_entry(int32_t ca, int32_t cb) const {
    if constexpr (SM) {
      const uint32_t ka = ca >= 0 ? ctab[ca] : 4u, kb = cb >= 0 ? ctab[cb] : 4u;
      return l16::selnib(ka, 0) | (8u << 4) | (l16::selnib(kb, 4) << 8) | (8u << 12);
    } else {
      // table rows: characters 0..255, row 256 (all zero) for out-of-range columns
      return (uint32_t)(ca >= 0 ? ca : 256) | ((uint32_t)(cb >= 0 ? cb : 256) << 16);
    }
  }
  // Copy the characters of local columns [c0, c0 + 32) into the byte ring: 4-byte granules
  // w0 + lane, lanes 0..8 (w0 = (col0 + c0) / 4); the last granule of b is zero-filled past its
  // end.  Columns outside this rank's range land in the ring too and are never read as such.
  __device__ __forceinline__ void copy_chars(int lane, int w0, int wlim, int btot) const {
    const int w = w0 + lane;
    if (lane < 9 && w < wlim) {
      const int rem = btot - 4 * w;
      cp_async_4(chr + ((4 * w) & (l16::kChr - 1)), bsrc + 4 * w, rem < 4 ? rem : 4);
    }
    cp_async_commit();
  }
  __device__ __forceinline__ int32_t leftval(const FillParams& p, int64_t i) const {
    if (i >= 0) return p.lcol_in != nullptr ? __ldcg(static_cast<const int32_t*>(p.lcol_in) + i) : 0;
    return 0;   // table row 0 (i = -1) and the virtual rows above it: LCS boundary 0
  }

  // Per-strip loop state in registers (opaque copies of FillParams fields and per-lane pointers,
  // advanced by one chunk per iteration).
  struct Links {
    const uint64_t* gprev;   // strip s-1's boundary row (base)
    uint64_t* gmine;         // strip s's boundary row (base)
    int32_t* stg;            // bottom staging row (packed, relative to the chunk's base)
    int32_t* tstg;           // top staging row (relative lo halves)
    uint32_t ep32;
    int cols, col0, btot, wlim;
    const uint64_t* pf;      // prefetch source of chunk k+1: gprev + 32(k+1) + 2 lane
    uint64_t* pub;           // publish target of chunk k-1-ELAG: gmine + 32(k-1-ELAG) + lane
    int32_t* lrow;           // last_row + 32(k-1-ELAG) + lane (BS 3)
  };

  // Top pairs of chunk k (columns 32k + lane), validated before the chunk's steps run.
  template <int TS>
  __device__ __forceinline__ bool acquire_top(const FillParams& p, int lane, int k, int NQ, const Links& lk,
                                              Control* ctl) {
    if (TS == 0 || k >= NQ) return true;   // past the last chunk the injections are 0 (chunk())
    tp = pbuf[lane];   // copied during the previous chunk (k = 0: at strip start)
    if (__all_sync(0xffffffffu, (uint32_t)(tp >> 32) == lk.ep32)) return true;
    const uint64_t* src = lk.gprev + 32 * k + lane;
    const long long t0 = clock64();
    Backoff w;
    int spins = 0;
    while (true) {
      if ((uint32_t)(tp >> 32) != lk.ep32) tp = ad_ld_gpu(src);
      if (__all_sync(0xffffffffu, (uint32_t)(tp >> 32) == lk.ep32)) break;
      if (++spins > p.spin_polls && !w.tick(ctl, p.timeout_ns)) return false;
    }
    wait_top += clock64() - t0;
    return true;
  }
  // chunk k+1's top pairs -> pbuf (lanes 0..15, 16 bytes each)
  template <int TS>
  __device__ __forceinline__ void prefetch_top(int lane, int k1, int NQ, const Links& lk) {
    if (TS == 2 && k1 < NQ && lane < 16) l16::cp_async_cg16(pbuf + 2 * lane, lk.pf);
    cp_async_commit();
  }

  // Bottom chunk j (columns 32j + lane): staged by lane 31 during the chunk that produced it.
  // BS 2: boundary row of this strip (pairs); 3: the last_row output; 0: nothing.
  template <int BS>
  __device__ __forceinline__ void publish_bottom(int lane, int j, int NQ, const Links& lk) {
    if (BS == 0 || j < 0 || j >= NQ) return;
    __syncwarp();
    const int32_t v = (int32_t)((uint32_t)lk.stg[lane] >> 16) + base;
    if (BS == 2) {
      asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(lk.pub), "l"(ad_pair((uint32_t)v, lk.ep32)) : "memory");
    } else {
      if (32 * j + lane < lk.cols) *lk.lrow = v;
    }
  }

  // Keep relative values small: subtract K = (lane 0's A row 0) - 4096 from every register.
  // Every value the warp holds is >= v0 - (64P rows + 64E columns + 2 steps of fifo age) >
  // v0 - 4096 (P, E <= 8), and <= v0 + 64P + 8 chunks of growth < 8192: 16 bits suffice.
  __device__ __forceinline__ void rebase() {
    static_assert(64 * P + 64 * E + 64 <= 4096, "rebase margin");
    const int32_t v0 = (int32_t)(__shfl_sync(0xffffffffu, h[0], 0) & 0xFFFFu);
    const int32_t K = v0 > 8192 ? v0 - 4096 : 0;
    if (K == 0) return;   // warp-uniform
    const uint32_t nk = (uint32_t)(0x10000 - K) & 0xFFFFu;
    const uint32_t nk2 = nk | (nk << 16);
#pragma unroll
    for (int q = 0; q < P; ++q) h[q] = __vadd2(h[q], nk2);
#pragma unroll
    for (int d = 0; d < E; ++d) fifo[d] = __vadd2(fifo[d], nk2);
    U0p = __vadd2(U0p, nk2);
    base += K;
  }

  // One chunk = 32 steps tau = 32k - E + su in 4 groups of 8.
  template <bool SM, int TS>
  __device__ __forceinline__ void chunk(const int lane, const int k, const int NQ, const Links& lk, const int w0) {
    const int lane_off = lane * E;
    // chunk k's top row (relative) -> shared memory; lane 31 injects it one group ahead.  Past
    // the last chunk (k >= NQ) tp keeps chunk NQ-1's pair: a top value within 32 columns of
    // column n-1, <= the rows' own past-the-end values (they stay constant) and close enough to
    // them to survive later rebases (a constant 0 would wrap below the rebased range)
    lk.tstg[lane] = max((int32_t)(uint32_t)tp - base, 0);
    __syncwarp();
    uint32_t injq[8];
    {
      const uint4 i0 = reinterpret_cast<const uint4*>(lk.tstg)[0];
      const uint4 i1 = reinterpret_cast<const uint4*>(lk.tstg)[1];
      injq[0] = i0.x; injq[1] = i0.y; injq[2] = i0.z; injq[3] = i0.w;
      injq[4] = i1.x; injq[5] = i1.y; injq[6] = i1.z; injq[7] = i1.w;
    }
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      if (g == 1) {
        // column ring: the entry of column 32(k+1) + lane (first read by group 3's look-ahead:
        // placed mid-chunk so its two dependent LDS hide behind the steps), then the
        // characters of columns 32(k+2) ..
        const int c = 32 * (k + 1) + lane;
        const int slot = c & (l16::kRing - 1);
        const uint32_t v = ring_entry<SM>(chr_at(lk.cols, lk.col0, c), chr_at(lk.cols, lk.col0, c - 32 * E));
        ring[slot] = v;
        if (slot < 8) ring[slot + l16::kRing] = v;
        copy_chars(lane, w0, lk.wlim, lk.btot);
      }
      if (g == l16::kPfGroup) prefetch_top<TS>(lane, k + 1, NQ, lk);
      const int tau0 = 32 * k - E + 8 * g;
      uint32_t injn[8];
      if (g < 3) {
        const uint4 i0 = reinterpret_cast<const uint4*>(lk.tstg + 8 * g + 8)[0];
        const uint4 i1 = reinterpret_cast<const uint4*>(lk.tstg + 8 * g + 8)[1];
        injn[0] = i0.x; injn[1] = i0.y; injn[2] = i0.z; injn[3] = i0.w;
        injn[4] = i1.x; injn[5] = i1.y; injn[6] = i1.z; injn[7] = i1.w;
      }
      uint32_t bv[8];
      // the next group's selectors (group 0 of chunk k+1: its ring entries were all written by
      // the start of this chunk), loaded a group ahead so the LDS latency stays off the steps
      uint32_t sn[8];
      if (g == 3) __syncwarp();   // group 1's ring entries are read by this look-ahead
      {
        const uint32_t* rn = ring + ((tau0 + 8 - lane_off) & (l16::kRing - 1));
#pragma unroll
        for (int u = 0; u < 8; ++u) sn[u] = rn[u];
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t s = sq[u];
        uint32_t mk[P];
        if constexpr (SM) {
#pragma unroll
          for (int q = 0; q < P; ++q) mk[q] = l16::prmt(tabA[q], tabB[q], s);
        } else {
          const uint32_t wa = mtab[(s & 0xFFFFu) * 32 + lane] & 0xFFu;
          const uint32_t wb = mtab[(s >> 16) * 32 + lane] >> 8;
          const uint32_t comb = l16::imad(wb, 65536u, wa);   // A bits 0..7, B bits 16..23
#pragma unroll
          for (int q = 0; q < P; ++q) mk[q] = (comb >> q) & 0x00010001u;
        }
        const uint32_t U0 = fifo[E - 1];
        uint32_t U = U0, UL = U0p;
        uint32_t nw[P];
#pragma unroll
        for (int q = 0; q < P; ++q) {
          const uint32_t X = l16::imad(mk[q], one, UL);
          const uint32_t v = __vimax3_u16x2(U, h[q], X);
          UL = h[q];
          U = v;
          nw[q] = v;
        }
        U0p = U0;
        bv[u] = nw[P - 1];
        const uint32_t sv = l16::prmt(nw[P - 1], injq[u], ssel);
        const uint32_t rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
        for (int d = E - 1; d > 0; --d) fifo[d] = fifo[d - 1];
        fifo[0] = rv;
#pragma unroll
        for (int q = 0; q < P; ++q) h[q] = nw[q];
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        if (g < 3) injq[u] = injn[u];
        sq[u] = sn[u];
      }
      if (lane == 31) {
        uint4* d = reinterpret_cast<uint4*>(lk.stg + 8 * g);
        d[0] = make_uint4(bv[0], bv[1], bv[2], bv[3]);
        d[1] = make_uint4(bv[4], bv[5], bv[6], bv[7]);
      }
    }
  }

  template <bool SM, int TS, int BS>
  __device__ __forceinline__ bool strip(const FillParams& p, int lane, int NQ, Links lk, Control* ctl) {
    const int K = NQ + ELAG;
    const bool trace = l16::opq(p.trace != nullptr ? 1 : 0) != 0;
    lk.cols = l16::opq(p.cols);
    lk.col0 = l16::opq(p.col0);
    lk.btot = l16::opq(p.cols_total);
    lk.wlim = (lk.btot + 3) >> 2;
    lk.ep32 = (uint32_t)l16::opq((int)lk.ep32);
    lk.pf = l16::opqp(lk.gprev + 32 + 2 * lane);
    lk.pub = l16::opqp(lk.gmine + lane - 32 * (1 + ELAG));
    lk.lrow = l16::opqp(static_cast<int32_t*>(p.last_row) + lane - 32 * (1 + ELAG));
    int w0 = ((lk.col0 + 64) >> 2);   // granule of column 32(k+2) at k = 0 (8 granules per chunk)
    for (int k = 0; k < K; ++k) {
      publish_bottom<BS>(lane, k - 1 - ELAG, NQ, lk);   // staged during chunk k-1 (its base)
      // every 8 chunks (a chunk adds at most 32 to any value: 16 bits keep > 60000 of headroom)
      if ((k & 7) == 0 && k > 0) rebase();
      // chunk k-1's copies (characters of columns 32(k+1).., chunk k's top pairs) have landed
      l16::cp_async_wait_all();
      __syncwarp();
      if (!acquire_top<TS>(p, lane, k, NQ, lk, ctl)) return false;
      if (trace && k == 0) t_first = globaltimer_ns();
      chunk<SM, TS>(lane, k, NQ, lk, w0);
      w0 += 8;
      lk.pf += 32;
      lk.pub += 32;
      lk.lrow += 32;
    }
    l16::cp_async_wait_all();
    publish_bottom<BS>(lane, K - 1 - ELAG, NQ, lk);
    return true;
  }
  template <bool SM>
  __device__ __forceinline__ bool strip_roles(const FillParams& p, int lane, int NQ, int TS, int BS, const Links& lk,
                                              Control* ctl) {
    if (TS == 2) {
      if (BS == 2) return strip<SM, 2, 2>(p, lane, NQ, lk, ctl);
      if (BS == 3) return strip<SM, 2, 3>(p, lane, NQ, lk, ctl);
      return strip<SM, 2, 0>(p, lane, NQ, lk, ctl);
    }
    if (BS == 2) return strip<SM, 0, 2>(p, lane, NQ, lk, ctl);
    if (BS == 3) return strip<SM, 0, 3>(p, lane, NQ, lk, ctl);
    return strip<SM, 0, 0>(p, lane, NQ, lk, ctl);
  }
};

// WPC independent warps per CTA: each claims its own strips; packing them into one CTA pins warp
// w to SM sub-partition w % 4 (one-warp CTAs could share a sub-partition and pace the pipeline)
template <int P, int E, int WPC>
__global__ void __launch_bounds__(32 * WPC, 1) lcs16_kernel(const FillParams p) {
  using LW = L16Warp<P, E>;
  constexpr int SH = LW::SH;
  __shared__ __align__(16) uint32_t ring_sh[WPC][l16::kRing + 8];
  __shared__ __align__(16) uint8_t chr_sh[WPC][l16::kChr];
  __shared__ __align__(16) uint64_t pbuf_sh[WPC][32];
  __shared__ __align__(16) int32_t stg_sh[WPC][32];
  __shared__ __align__(16) int32_t tstg_sh[WPC][32];
  __shared__ uint8_t ctab_sh[WPC][256];
  __shared__ int one_sh[WPC];
  // per warp: the match table of the table path (257 characters x 32 lanes x 16-bit masks)
  extern __shared__ __align__(16) uint8_t l16_dyn[];

  Control* ctl = static_cast<Control*>(p.ctl);
  const int lane = threadIdx.x & 31;
  const int wid = threadIdx.x >> 5;
  const int n = p.cols;
  const int NQ = (n + 31) / 32;
  uint32_t* ring = ring_sh[wid];
  uint8_t* ctab = ctab_sh[wid];
  uint16_t* mtab = reinterpret_cast<uint16_t*>(l16_dyn + wid * l16::kDynPerWarp);
  if (lane == 0) one_sh[wid] = p.one;
  __syncwarp();

  const bool worker = (int)(blockIdx.x * WPC + wid) < p.workers;
  while (worker) {
    int s = 0;
    if (lane == 0) {
      s = (int)atomicAdd(&ctl->claim, 1u);
      if (ld_volatile_u32(&ctl->abort)) s = INT_MAX;
    }
    s = __shfl_sync(0xffffffffu, s, 0);
    if (s >= p.nstrips) break;
    const int64_t top = p.row0 + (int64_t)s * SH;
    const bool last_strip = (s == p.nstrips - 1);

    LW lw;
    bool ok = true;
    // multi-GPU: rank g-1's right column of this strip and the previous strip's last row
    if (p.lcol_in != nullptr) ok = window_consume_wait(p, s, ctl);
    // rows of this lane: A = top + lane*P + q, B = top + 32P + lane*P + q
    const int64_t rowA = top + (int64_t)lane * P, rowB = rowA + 32 * P;
    int32_t chA[P], chB[P];
#pragma unroll
    for (int q = 0; q < P; ++q) {
      chA[q] = rowA + q >= 0 ? (int32_t)static_cast<const uint8_t*>(p.a)[rowA + q] : -1;
      chB[q] = rowB + q >= 0 ? (int32_t)static_cast<const uint8_t*>(p.a)[rowB + q] : -1;
    }
    // base = the corner LCS(top-1, -1): every value of the strip is >= it (monotone).  Registers
    // start at the left boundary (column -1): h = the lane's rows, U / UL of pair 0 = the rows
    // above them (lane k-1's last rows; lane 0: the corner and band A's last row)
    lw.base = lw.leftval(p, top - 1);
#pragma unroll
    for (int q = 0; q < P; ++q) lw.h[q] = l16::pack(lw.leftval(p, rowA + q) - lw.base, lw.leftval(p, rowB + q) - lw.base);
    const uint32_t up = l16::pack(lw.leftval(p, rowA - 1) - lw.base, lw.leftval(p, rowB - 1) - lw.base);
#pragma unroll
    for (int d = 0; d < E; ++d) lw.fifo[d] = up;
    lw.U0p = up;
    if (p.lcol_in != nullptr) {   // every left value of the strip is in registers: release the slot
      __syncwarp();
      if (lane == 0 && ok) window_consume_ack(p, s);
    }
    lw.one = ad_ld_smem_i32(&one_sh[wid]);
    lw.ssel = lane == 31 ? 0x1054u : 0x3210u;
    lw.ring = ring;
    lw.chr = chr_sh[wid];
    lw.ctab = ctab;
    lw.mtab = mtab;
    lw.pbuf = pbuf_sh[wid];
    // distinct row characters of the warp: <= 4 -> codes 0..3 (PRMT path), else table path
    for (int j = 0; j < 8; ++j) ctab[8 * lane + j] = 0xFF;
    __syncwarp();
#pragma unroll
    for (int q = 0; q < P; ++q) {
      if (chA[q] >= 0) ctab[chA[q]] = 0;
      if (chB[q] >= 0) ctab[chB[q]] = 0;
    }
    __syncwarp();
    uint32_t pb = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) pb |= (ctab[8 * lane + j] == 0 ? 1u : 0u) << j;
    const int cnt = __popc(pb);
    int pre = cnt;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const int t = __shfl_up_sync(0xffffffffu, pre, off);
      if (lane >= off) pre += t;
    }
    const bool small = __shfl_sync(0xffffffffu, pre, 31) <= 4;
    __syncwarp();
    if (small) {
      const int base0 = pre - cnt;
#pragma unroll
      for (int j = 0; j < 8; ++j)
        ctab[8 * lane + j] = ((pb >> j) & 1u) ? (uint8_t)(base0 + __popc(pb & ((1u << j) - 1u))) : (uint8_t)4;
      __syncwarp();
#pragma unroll
      for (int q = 0; q < P; ++q) {
        const uint32_t ka = chA[q] >= 0 ? ctab[chA[q]] : 4u, kb = chB[q] >= 0 ? ctab[chB[q]] : 4u;
        lw.tabA[q] = ka < 4 ? 1u << (8 * ka) : 0u;
        lw.tabB[q] = kb < 4 ? 1u << (8 * kb) : 0u;
      }

    } else {
      for (int c = 0; c < 257; ++c) mtab[c * 32 + lane] = 0;
      __syncwarp();
#pragma unroll
      for (int q = 0; q < P; ++q) {
        if (chA[q] >= 0) mtab[chA[q] * 32 + lane] |= (uint16_t)(1u << q);
        if (chB[q] >= 0) mtab[chB[q] * 32 + lane] |= (uint16_t)(256u << q);
        lw.tabA[q] = 0;
        lw.tabB[q] = 0;
      }
    }
    __syncwarp();
    // byte ring: columns [-32(E+1), 64) loaded synchronously; column ring: columns up to 31
    for (int c = -32 * (E + 1) + lane; c < 64; c += 32)
      if ((unsigned)c < (unsigned)n) lw.chr[(p.col0 + c) & (l16::kChr - 1)] = static_cast<const uint8_t*>(p.b)[p.col0 + c];
    __syncwarp();
    for (int q = -E - 1; q <= 0; ++q) {
      const int c = 32 * q + lane;
      const int32_t ca = lw.chr_at(n, p.col0, c), cb = lw.chr_at(n, p.col0, c - 32 * E);
      const uint32_t v = small ? lw.template ring_entry<true>(ca, cb) : lw.template ring_entry<false>(ca, cb);
      const int slot = c & (l16::kRing - 1);
      ring[slot] = v;
      if (slot < 8) ring[slot + l16::kRing] = v;
    }
    __syncwarp();
#pragma unroll
    for (int u = 0; u < 8; ++u) lw.sq[u] = ring[((-E - lane * E) & (l16::kRing - 1)) + u];   // chunk 0, group 0


    const int TS = (s > 0 && !(p.debug & 2)) ? 2 : 0;   // debug 2: no strip handoff (timing only)
    const int BS = last_strip ? (p.last_row != nullptr ? 3 : 0) : 2;
    const uint64_t gt0 = globaltimer_ns();
    const long long ck0 = clock64();
    lw.wait_top = 0;
    lw.t_first = 0;
    typename LW::Links lk;
    lk.gprev = static_cast<const uint64_t*>(p.bnd) + (int64_t)(s - 1) * p.bnd_stride;
    lk.gmine = static_cast<uint64_t*>(p.bnd) + (int64_t)s * p.bnd_stride;
    lk.stg = stg_sh[wid];
    lk.tstg = tstg_sh[wid];
    lk.ep32 = (uint32_t)p.epoch;
    lw.tp = 0;
    lw.bsrc = static_cast<const uint8_t*>(p.b);
    if (TS == 2) {   // chunk 0's top pairs
      lk.pf = lk.gprev + 2 * lane;
      lw.template prefetch_top<2>(lane, 0, NQ, lk);
    }
    ok = ok && (small ? lw.template strip_roles<true>(p, lane, NQ, TS, BS, lk, ctl)
                      : lw.template strip_roles<false>(p, lane, NQ, TS, BS, lk, ctl));
    if (p.trace != nullptr && lane == 0) {
      uint64_t* tr = p.trace + (int64_t)s * 8;
      tr[0] = gt0;
      tr[1] = globaltimer_ns();
      tr[2] = (uint64_t)(clock64() - ck0);
      tr[3] = (uint64_t)lw.wait_top;
      tr[4] = lw.t_first;   // globaltimer when chunk 0's top row was in (pipeline fill ends)
      uint32_t smid, warpid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      asm volatile("mov.u32 %0, %%warpid;" : "=r"(warpid));
      tr[5] = ((uint64_t)smid << 32) | warpid;
      tr[6] = 0;
      tr[7] = 0;
    }
    // right column = the final registers (rows keep their column n-1 value past the end); into
    // rank g+1's window once rank g+1 has released this slot
    if (p.rcol_out != nullptr) {
      int pw = 0;
      if (lane == 0) pw = ok && window_produce_wait(p, s, ctl);
      ok = __shfl_sync(0xffffffffu, pw, 0) != 0;
    }
    if (ok) {
#pragma unroll
      for (int q = 0; q < P; ++q) {
#pragma unroll
        for (int hb = 0; hb < 2; ++hb) {
          const int64_t i = (hb ? rowB : rowA) + q;
          const int32_t v = (int32_t)(hb ? (lw.h[q] >> 16) : (lw.h[q] & 0xFFFFu)) + lw.base;
          if (i >= 0 && i < p.rows) {
            if (p.last_col != nullptr) static_cast<int32_t*>(p.last_col)[i] = v;
            if (p.rcol_out != nullptr) static_cast<int32_t*>(p.rcol_out)[i] = v;
            if (i == p.rows - 1 && p.score != nullptr && p.is_last_rank) *static_cast<int32_t*>(p.score) = v;
          }
        }
      }
      if (p.rcol_out != nullptr) __threadfence_system();
    }
    __syncwarp();
    if (p.rflag_out != nullptr && lane == 0 && ok) {
      __threadfence_system();
      st_release_sys(p.rflag_out + s, (p.wepoch << 32) | 1u);
    }
  }
  if (lane == 0) {
    __threadfence();
    const unsigned d = atomicAdd(&ctl->done, 1u);
    if (d == gridDim.x * WPC - 1) {
      atomicExch(&ctl->claim, 0u);
      atomicExch(&ctl->done, 0u);
    }
  }
}

template <int P, int E>
cudaError_t lcs16_launch(const FillParams& p, int warps, cudaStream_t s) {
  constexpr int WPC = 4;
  constexpr size_t dyn = WPC * l16::kDynPerWarp;
  FillParams q = p;
  q.workers = warps;
  static bool attr = false;   // > 48 KB of dynamic shared memory: opt in once
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(lcs16_kernel<P, E, WPC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  lcs16_kernel<P, E, WPC><<<(warps + WPC - 1) / WPC, 32 * WPC, dyn, s>>>(q);
  return cudaGetLastError();
}

// Compiled geometries (P pairs = 2P rows per lane, E steps of lane lag); `warps` persistent
// strip workers (rounded up to whole 4-warp CTAs).  b must be 4-byte aligned (cp.async granules).
cudaError_t launch_lcs16(const FillParams& p, int P, int E, int warps, cudaStream_t s) {
#define LDDP_L16_GEOM(PP, EE) \
  if (P == PP && E == EE) return lcs16_launch<PP, EE>(p, warps, s);
  LDDP_L16_GEOMS
#undef LDDP_L16_GEOM
  return cudaErrorInvalidValue;
}
bool lcs16_compiled(int P, int E) {
#define LDDP_L16_GEOM(PP, EE) \
  if (P == PP && E == EE) return true;
  LDDP_L16_GEOMS
#undef LDDP_L16_GEOM
  return false;
}

}  // namespace lddp
