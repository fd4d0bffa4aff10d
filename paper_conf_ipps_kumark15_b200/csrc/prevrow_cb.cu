// prevrow_cb.cu -- previous-row-only ("Horizontal", t = i) category, column-block persistent
// kernel [L180-L195], Fig. 2(b).  The default prev-row kernel when the grid is 32-bit, W % 4 == 0
// and the column blocks fit co-resident (cooperative launch); prevrow.cu is the fallback.
//
// Every cell of row i depends only on row i-1 (contributing set within {UL, U, UR}), so the
// degree of parallelism is the row width in every iteration [L184].  The paper launches one
// kernel per row [L184], [L251]; here ONE cooperative launch fills the whole table:
//
//  * Warp q owns the column block [q*BW, (q+1)*BW) for ALL rows: its DP state never leaves the
//    register file.  Lane l holds VP consecutive columns of the extended window
//    [q*BW - HB, (q+1)*BW + HB), EXT = 32*VP = BW + 2*HB.
//  * Bands of HB rows.  Within a band the warp recomputes the two HB-column halos itself (the
//    TRAPEZOID: garbage entering from the window's outer edges advances one column per row, so
//    after HB rows it has not reached the block's own columns).  At each band boundary the warp
//    publishes the HB own columns at each edge and replaces its halos with the neighbours'
//    published edges: case-2 two-way halo of Table II [L265-L274], ([L193-L195]), one exchange
//    per HB rows instead of one per row.
//  * Edge exchange = (value, tag) 64-bit pairs in global memory (single-copy atomic): the
//    consumer polls the data itself, no flag, no fence.  Tag = (fill epoch mod 2048) << 20 | band + 1
//    (bit 31 set for multi-GPU fills, whose epoch is the rank-consistent fill count).
//  * Multi-GPU (lddp_fill_multi): each rank owns a block-aligned column strip; the strip's outer
//    blocks also push their edges into the neighbour ranks' comm windows (system-scope stores over
//    NVLink) and take their halos from their own window -- the same two-way exchange, one band
//    at a time, across GPUs (Table II case 2 [L265-L274], [L193-L195]).
//  * Cost rows (the HBM stream, 4 B/cell) flow through a per-warp D-row shared-memory ring
//    filled by 16-byte cp.async (LDGSTS.128, L1 bypass; 8-byte when VP % 4 != 0), D-1 rows ahead
//    of the row being computed; every lane copies exactly the columns it later reads, so the ring
//    needs no warp synchronisation at all.  (MODE 1 / 2: bulk / 2-D tensor TMA instead --
//    measured slower, kept selectable.)
//  * Table edges: out-of-table cells are never forced; column 0's UL and column W-1's UR take
//    f's boundary value (the edge warps would otherwise pace everyone through the exchange).
//  * The last band writes last_row and the row minimum (score).
//  * Measured and rejected geometries (lane ghosts, 2-D tensor TMA, VP 8 / HB 32, 32-row rings)
//    are no longer built (DESIGN.md §5.2 has their numbers).
#include <cstdint>
#include <climits>
#include "cellfn.cuh"
#include "params.h"
#include "sync.cuh"
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cstring>
#include <type_traits>

namespace lddp {

__device__ __forceinline__ void cb_cp16(void* dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cb_cp16s(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cb_tma_row(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ bool cb_bar_ready(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}
// 2-D tensor TMA of one row group: box {EXT columns, kCbRG rows} at (x, y); out-of-table
// elements (negative x, x >= W, y >= H) are zero-filled by the TMA unit.
constexpr int kCbRG = 32;   // rows per tensor TMA
constexpr int kCbNG = 3;    // row groups in flight per warp (ring = kCbNG * kCbRG rows)
__device__ __forceinline__ void cb_tma_tile(uint32_t dst, const CUtensorMap* tmap, int x, int y, uint32_t bar,
                                            uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(x), "r"(y), "r"(bar)
      : "memory");
}

// Bulk (TMA) row stream state of one warp: lane 0 issues one cp.async.bulk per row for the
// in-table part of the warp's extended window; completion on one mbarrier per ring slot.
struct CbBulk {
  uint32_t dst0;      // shared address of slot 0's first in-table column
  uint32_t bytes;     // in-table bytes of the window (multiple of 16)
  uint32_t bar0;      // shared address of slot 0's mbarrier
  const void* src0;   // global address of row 0's first in-table column
  int irow, islot;    // next row to issue and its slot (MODE 2: next row group's first row)
  int x0;             // MODE 2: first column of the warp's window (may be negative)
  uint32_t cpar;      // phase parity of the slot being consumed
};

__device__ __forceinline__ void cb_cp8s(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
// lane segments: 16 bytes (4 columns) when VP % 4 == 0, else 8 bytes (2 columns)
template <int VP> constexpr int kCbSeg = (VP % 4 == 0) ? 4 : 2;
template <int VP> constexpr int kCbNSeg = VP / kCbSeg<VP>;
template <int VP, class G>
__device__ __forceinline__ void cb_issue(uint32_t idst, const G* const (&src)[kCbNSeg<VP>], const uint32_t (&ssz)[kCbNSeg<VP>],
                                         int64_t ioff) {
#pragma unroll
  for (int s = 0; s < kCbNSeg<VP>; ++s) {
    if constexpr (kCbSeg<VP> == 4) cb_cp16s(idst + 16 * s, src[s] + ioff, ssz[s]);
    else cb_cp8s(idst + 8 * s, src[s] + ioff, ssz[s]);
  }
}
template <int VP, class G>
__device__ __forceinline__ void cb_lds(const G* gs, G (&g)[VP]) {
#pragma unroll
  for (int s = 0; s < kCbNSeg<VP>; ++s) {
    if constexpr (kCbSeg<VP> == 4) {
      const int4 t = *reinterpret_cast<const int4*>(gs + 4 * s);
      g[4 * s] = t.x; g[4 * s + 1] = t.y; g[4 * s + 2] = t.z; g[4 * s + 3] = t.w;
    } else {
      const int2 t = *reinterpret_cast<const int2*>(gs + 2 * s);
      g[2 * s] = t.x; g[2 * s + 1] = t.y;
    }
  }
}

__device__ __forceinline__ void cb_st_pair2(uint64_t* p, uint64_t a, uint64_t b) {
  asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void cb_ld_pair2(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
// system scope: edge pairs exchanged with the neighbour GPUs' windows (NVLink peer memory)
__device__ __forceinline__ void cb_st_pair2_sys(uint64_t* p, uint64_t a, uint64_t b) {
  asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void cb_ld_pair2_sys(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.sys.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

// Table-edge masks of an edge warp (see cb_band): lv' = (lv & lA) | lO, UR'[v] = (UR & rA[v]) | rO[v]
template <int VP>
struct CbEdge {
  uint32_t lA, lO;
  uint32_t rA[VP], rO[VP];
};
template <class T>
__device__ __forceinline__ T cb_fix(T x, uint32_t A, uint32_t O) {
  static_assert(sizeof(T) == 4, "32-bit cells");
  uint32_t u;
  memcpy(&u, &x, 4);
  u = (u & A) | O;
  memcpy(&x, &u, 4);
  return x;
}

// One band of nr <= HB rows.  OUT: this lane holds out-of-table columns (their value is f's
// boundary value in every row: one extra select per cell, taken only by the two edge blocks'
// edge lanes -- warp-uniform for every other warp).
template <class F, int VP, int D, bool TABLE, bool OUT, int MODE>
__device__ __forceinline__ void cb_band(CbBulk& bk, const CUtensorMap* tmap, const int lane, const FillParams& p, typename F::T (&cur)[VP], typename F::GridT (&g)[VP],
                                        const int nr, const int64_t r0,
                                        const typename F::GridT* ring, int& cslot, uint32_t& idst, int& ileft,
                                        int64_t& ioff, const int64_t pitch,
                                        const typename F::GridT* const (&src)[kCbNSeg<VP>], const uint32_t (&ssz)[kCbNSeg<VP>],
                                        const CbEdge<VP>& ed, const int e0,
                                        const int j0, const int BW) {
  using T = typename F::T;
  using G = typename F::GridT;
  constexpr int EXT = 32 * VP;
  const uint32_t ibeg = smem_u32(ring), iend = ibeg + (D - 1) * EXT * 4;
#pragma unroll 2
  for (int r = 0; r < nr; ++r) {
    // issue row + D - 1 into the slot consumed last (32-bit shared address, wraps at the ring end).
    // The global address is formed into a fresh register from the lane's row-0 pointer and a
    // running element offset: updating the LDGSTS address register in place made the next row
    // wait on the copy's register read (long-scoreboard stalls on the pointer increment).
    if constexpr (MODE == 2) {
      // tensor rows arrive in groups of kCbRG: nothing to issue per row
    } else if constexpr (MODE == 1) {
      if (lane == 0 && bk.irow < p.rows)
        cb_tma_row(bk.dst0 + bk.islot * EXT * 4, static_cast<const char*>(bk.src0) + (int64_t)bk.irow * pitch * 4,
                   bk.bytes, bk.bar0 + bk.islot * 8);
      ++bk.irow;
      bk.islot = (bk.islot + 1 == D) ? 0 : bk.islot + 1;
    } else {
      if (ileft > 0) cb_issue<VP>(idst, src, ssz, ioff);
      ioff += pitch;
      --ileft;
      idst = (idst == iend) ? ibeg : idst + EXT * 4;
      cp_async_commit();
      cp_async_wait_group<D - 2>();    // the NEXT row's group has landed: load it now, use it next row
    }
    G gn[VP];
    cslot = (cslot + 1 == D) ? 0 : cslot + 1;
    if constexpr (MODE == 1) {
      if (cslot == 0) bk.cpar ^= 1u;
      if (r0 + r + 1 < p.rows)
        while (!cb_bar_ready(bk.bar0 + cslot * 8, bk.cpar)) {
        }
    }
    if constexpr (MODE == 2) {
      if (cslot % kCbRG == 0) {
        // entering a new row group: the previous group is fully read -> refill its slot with the
        // group kCbNG ahead (one 2-D tensor TMA of kCbRG rows x EXT columns), then wait for this one
        const int gnew = cslot / kCbRG;
        const int gold = (gnew == 0 ? kCbNG : gnew) - 1;
        if (cslot == 0) bk.cpar ^= 1u;
        if (lane == 0) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          cb_tma_tile(bk.dst0 + gold * kCbRG * EXT * 4, tmap, bk.x0, bk.irow, bk.bar0 + gold * 8, kCbRG * EXT * 4);
        }
        bk.irow += kCbRG;
        if (r0 + r + 1 < p.rows)
          while (!cb_bar_ready(bk.bar0 + gnew * 8, bk.cpar)) {
          }
      }
    }
    cb_lds<VP>(ring + cslot * EXT, gn);
    const int64_t row = r0 + r;
    T lv = __shfl_up_sync(0xffffffffu, cur[VP - 1], 1);   // lane 0: own value (halo garbage)
    const T rv = __shfl_down_sync(0xffffffffu, cur[0], 1);
    // Table edges (OUT warps only): out-of-table cells are never forced; instead the two cells
    // that read them take f's boundary value as that neighbour -- column 0's UL (always v = 0:
    // e0 % 4 == 0) and column W-1's UR (v % 4 == 3 since W % 4 == 0).  Forcing every outside
    // cell every row put selects on the row chain and made the two edge warps -- which pace all
    // others through the halo exchange -- twice as slow as an interior warp.
    // The fix is one LOP3 per edge cell, (x & A) | O with per-lane masks set once (A = 0, O =
    // the boundary value's bits on the lane holding the table edge; A = ~0, O = 0 elsewhere):
    // selects here let the compiler serialise the two shuffles of a row pair behind them (C4
    // edge warps 108 vs 64 cycles per row, pacing every warp through the exchange).
    if (OUT) lv = cb_fix(lv, ed.lA, ed.lO);
    T nw_[VP];
#pragma unroll
    for (int v = 0; v < VP; ++v) {
      const T UL = (v > 0) ? cur[v - 1] : lv;
      const T U = cur[v];
      T UR = (v < VP - 1) ? cur[v + 1] : rv;
      if (OUT && (VP % 4 != 0 || (v & 3) == 3)) UR = cb_fix(UR, ed.rA[v], ed.rO[v]);
      typename F::OutT o;
      T x = F::f(U, UL, U, UR, typename F::RowCtx(0), typename F::ColCtx(0), g[v], row, p.col0 + e0 + v, p.param_c, o);
      nw_[v] = x;
      if (TABLE) {
        const int col = e0 + v;
        if (col >= j0 && col < j0 + BW && col < p.cols)
          static_cast<typename F::OutT*>(p.table)[row * p.table_pitch + col] = o;
      }
    }
#pragma unroll
    for (int v = 0; v < VP; ++v) {
      cur[v] = nw_[v];
      g[v] = gn[v];
    }
  }
}

template <class F, int VP, int HB, int D, bool TABLE, int MODE>
__global__ void __launch_bounds__(256) prevrow_cb_kernel(const FillParams p, const __grid_constant__ CUtensorMap tmap_) {
  const CUtensorMap* tmap = &tmap_;
  static_assert(MODE != 2 || D == kCbNG * kCbRG, "tensor mode: ring = kCbNG groups of kCbRG rows");
  using T = typename F::T;
  using G = typename F::GridT;
  static_assert(!(F::kMask & NB_L), "prev-row category: f must not read L");
  static_assert(sizeof(T) == 4 && sizeof(G) == 4, "32-bit cells and costs");
  static_assert(VP % 2 == 0 && HB % VP == 0, "8- or 16-byte lane segments; halos made of whole lanes");
  constexpr int EXT = 32 * VP;
  constexpr int BW = EXT - 2 * HB;
  constexpr int HL = HB / VP;            // lanes per halo
  static_assert(BW >= 2 * HB, "each edge publishes HB own columns");

  extern __shared__ __align__(128) unsigned char cb_smem[];
  const int lane = threadIdx.x & 31;
  const int wl = threadIdx.x >> 5;
  const int nw = blockDim.x >> 5;
  const int q = blockIdx.x * nw + wl;   // column block
  const int nb = p.nblocks;
  Control* ctl = static_cast<Control*>(p.ctl);
  const int W = p.cols;
  const int64_t H = p.rows;

  if (q < nb && H > 0) {
    G* ring = reinterpret_cast<G*>(cb_smem) + (size_t)wl * D * EXT + lane * VP;   // this lane's columns
    const int j0 = q * BW;
    const int e0 = j0 - HB + lane * VP;   // first column of this lane
    const G* cost = static_cast<const G*>(p.grid);
    // the table's columns in local coordinates: [clo, chi) (multi-GPU: this rank's strip is
    // [0, W) of the whole table [-col0, cols_total - col0); its halos reach into the neighbours')
    const int clo = -p.col0, chi = p.cols_total - p.col0;
    // out-of-table columns keep the boundary value of f in every row
    uint32_t omask = 0;
    T outv[VP];
#pragma unroll
    for (int v = 0; v < VP; ++v) {
      const int col = e0 + v;
      if (col < clo || col >= chi) omask |= 1u << v;
      outv[v] = col < clo ? F::left(p, 0) : F::right(p, 0);
    }
    bool anyout = __any_sync(0xffffffffu, omask != 0);
    if (p.debug & 16) anyout = false;   // development timing switches (wrong edge results)
    if (p.debug & 32) anyout = true;
    const bool lfix = (e0 == clo);                                             // column 0 at v = 0
    const int rfix = (chi - 1 >= e0 && chi - 1 < e0 + VP) ? (chi - 1 - e0) : -1;   // column W-1
    CbEdge<VP> ed;
    {
      const T lb = F::left(p, 0), rb = F::right(p, 0);
      uint32_t lbits, rbits;
      memcpy(&lbits, &lb, 4);
      memcpy(&rbits, &rb, 4);
      ed.lA = lfix ? 0u : ~0u;
      ed.lO = lfix ? lbits : 0u;
#pragma unroll
      for (int v = 0; v < VP; ++v) {
        ed.rA[v] = (rfix == v) ? 0u : ~0u;
        ed.rO[v] = (rfix == v) ? rbits : 0u;
        asm volatile("mov.b32 %0, %0;" : "+r"(ed.rA[v]));   // opaque: kept as LOP3 masks
        asm volatile("mov.b32 %0, %0;" : "+r"(ed.rO[v]));
      }
      asm volatile("mov.b32 %0, %0;" : "+r"(ed.lA));
      asm volatile("mov.b32 %0, %0;" : "+r"(ed.lO));
    }
    // 16-byte segments of this lane: all in or all out (W % 4 == 0, e0 % 4 == 0)
    constexpr int SEG = kCbSeg<VP>;
    uint32_t ssz[kCbNSeg<VP>];
    const G* src[kCbNSeg<VP>];
#pragma unroll
    for (int s = 0; s < kCbNSeg<VP>; ++s) {
      const int col = e0 + SEG * s;
      const bool in = col >= clo && col < chi;
      ssz[s] = in ? 4u * SEG : 0u;
      asm volatile("mov.b32 %0, %0;" : "+r"(ssz[s]));   // opaque: no per-row rematerialisation
      src[s] = cost + (in ? col : 0);
    }
    int ileft = (int)H;   // rows still to issue
    uint32_t idst = smem_u32(ring);
    int cslot = 0;
    int64_t pitch = p.grid_pitch;
    asm volatile("mov.b64 %0, %0;" : "+l"(pitch));   // held in a register, not reloaded per row
    int64_t ioff = 0;                                 // element offset of the next row to issue
    CbBulk bk{};
    if constexpr (MODE == 2) {
      const uint32_t wbase = smem_u32(reinterpret_cast<G*>(cb_smem) + (size_t)wl * D * EXT);
      bk.dst0 = wbase;
      bk.bar0 = smem_u32(reinterpret_cast<uint64_t*>(cb_smem + (size_t)nw * D * EXT * sizeof(G)) + wl * D);
      bk.x0 = j0 - HB;
      if (lane == 0) {
        for (int k = 0; k < kCbNG; ++k)
          asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bk.bar0 + 8 * k) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int k = 0; k < kCbNG; ++k)
          cb_tma_tile(wbase + k * kCbRG * EXT * 4, tmap, bk.x0, k * kCbRG, bk.bar0 + 8 * k, kCbRG * EXT * 4);
      }
      __syncwarp();
      bk.irow = kCbNG * kCbRG;
      bk.cpar = 0;
      while (!cb_bar_ready(bk.bar0, 0u)) {
      }
    } else if constexpr (MODE == 1) {
      const uint32_t wbase = smem_u32(reinterpret_cast<G*>(cb_smem) + (size_t)wl * D * EXT);
      const int cs = max(j0 - HB, 0), ce = min(j0 - HB + EXT, W);
      bk.dst0 = wbase + (uint32_t)(cs - (j0 - HB)) * 4u;
      bk.bytes = (uint32_t)(ce - cs) * 4u;
      bk.bar0 = smem_u32(reinterpret_cast<uint64_t*>(cb_smem + (size_t)nw * D * EXT * sizeof(G)) + wl * D);
      bk.src0 = cost + cs;
      if (lane == 0) {
        for (int k = 0; k < D; ++k)
          asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bk.bar0 + 8 * k) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      }
      __syncwarp();
      for (int k = 0; k < D - 1; ++k) {
        if (lane == 0 && k < H)
          cb_tma_row(bk.dst0 + k * EXT * 4, static_cast<const char*>(bk.src0) + (int64_t)k * pitch * 4, bk.bytes,
                     bk.bar0 + k * 8);
      }
      bk.irow = D - 1;
      bk.islot = D - 1;
      bk.cpar = 0;
      while (!cb_bar_ready(bk.bar0, 0u)) {
      }
    } else {
#pragma unroll 1
      for (int k = 0; k < D - 1; ++k) {
        if (ileft > 0) cb_issue<VP>(idst, src, ssz, ioff);
        ioff += pitch;
        --ileft;
        idst += EXT * 4;
        cp_async_commit();
      }
      cp_async_wait_group<D - 2>();
    }

    // costs of row 0 (the band loop loads row r+1 while computing row r)
    G g[VP];
    cb_lds<VP>(ring, g);

    // row -1 (virtual): f's top initialisation
    T cur[VP];
#pragma unroll
    for (int v = 0; v < VP; ++v) cur[v] = ((omask >> v) & 1u) ? outv[v] : F::top(p, p.col0 + e0 + v);   // global column

    // edge-pair tags: fill epoch (mod 2048) and band + 1 in disjoint bit fields -- every slot a fill
    // uses is rewritten by it, so a pair left by an earlier fill of this workspace never matches
  // (multi-GPU: the rank-consistent fill epoch, with bit 31 set, so the neighbours agree)
  const bool xrank = p.halo_in_l != nullptr || p.halo_in_r != nullptr;
  const uint32_t tag0 = xrank ? (0x80000000u | (uint32_t)(p.wepoch & 0x7FFu) << 20) : (uint32_t)(p.epoch & 0x7FFu) << 20;
    uint64_t* edges = reinterpret_cast<uint64_t*>(p.bnd);   // [nb][4 slots][2 sides][HB] pairs
    const bool lhalo = lane < HL, rhalo = lane >= 32 - HL;
    const bool ledge = lane >= HL && lane < 2 * HL;          // own columns [j0, j0 + HB)
    const bool redge = lane >= 32 - 2 * HL && lane < 32 - HL; // own columns [j0 + BW - HB, j0 + BW)

#pragma unroll 1
    for (int64_t r0 = 0; r0 < H; r0 += HB) {
      const int nr = (int)((H - r0 < HB) ? (H - r0) : HB);
      // development trace (LDDP_TRACE): per band of block `trace_chunks`, clock64 at entry / exit
#ifdef LDDP_CB_TRACE
      const bool trc = p.trace != nullptr && q == p.trace_chunks && lane == 0 && r0 / HB < 4096;
#else
      constexpr bool trc = false;   // the per-band checks cost ~8 % (measured on prevrow_hx)
#endif
      const long long tb0 = trc ? clock64() : 0;
      if (anyout)
        cb_band<F, VP, D, TABLE, true, MODE>(bk, tmap, lane, p, cur, g, nr, r0, ring, cslot, idst, ileft, ioff, pitch, src, ssz, ed, e0, j0, BW);
      else
        cb_band<F, VP, D, TABLE, false, MODE>(bk, tmap, lane, p, cur, g, nr, r0, ring, cslot, idst, ileft, ioff, pitch, src, ssz, ed, e0, j0, BW);
      if (trc) {
        p.trace[2 * (r0 / HB)] = (uint64_t)(clock64() - tb0);
      }
      if (r0 + HB >= H) break;   // last band: outputs below
      if (p.debug & 8) continue;   // development: no band exchange (wrong results; timing only)
      // ---- band boundary: publish own edges, take the neighbours' as halos
      const int band = (int)(r0 / HB);
      const uint32_t tag = tag0 | (((uint32_t)band + 1u) & 0xFFFFFu);
      uint64_t* mine = edges + ((size_t)q * 4 + (band & 3)) * 2 * HB;
      const int xslot = ((int)(p.wepoch & 1) * 4 + (band & 3)) * HB;   // multi-GPU window slot
      if (ledge || redge) {
        uint64_t* d = mine + (ledge ? 0 : HB) + (ledge ? (lane - HL) : (lane - (32 - 2 * HL))) * VP;
#pragma unroll
        for (int v = 0; v < VP; v += 2)
          cb_st_pair2(d + v, ((uint64_t)tag << 32) | (uint32_t)cur[v], ((uint64_t)tag << 32) | (uint32_t)cur[v + 1]);
        // multi-GPU: the strip's outer edges also go into the neighbour ranks' windows
        uint64_t* xo = nullptr;
        // (8 slots: fill parity x band mod 4 -- a rank may start fill k+1 while its neighbour still
        // reads fill k's last edges)
        if (ledge && q == 0 && p.halo_out_l != nullptr) xo = p.halo_out_l + xslot + (lane - HL) * VP;
        if (redge && q == nb - 1 && p.halo_out_r != nullptr) xo = p.halo_out_r + xslot + (lane - (32 - 2 * HL)) * VP;
        if (xo != nullptr) {
#pragma unroll
          for (int v = 0; v < VP; v += 2)
            cb_st_pair2_sys(xo + v, ((uint64_t)tag << 32) | (uint32_t)cur[v], ((uint64_t)tag << 32) | (uint32_t)cur[v + 1]);
        }
      }
      const int nbq = lhalo ? q - 1 : q + 1;
      // halo from the neighbour block of this GPU, or (strip edges) from the neighbour rank
      const bool xin = (lhalo && q == 0 && p.halo_in_l != nullptr) || (rhalo && q == nb - 1 && p.halo_in_r != nullptr);
      const bool need = (lhalo && q > 0) || (rhalo && q + 1 < nb) || xin;
      const uint64_t* s = nullptr;
      if (xin)
        s = lhalo ? p.halo_in_l + xslot + lane * VP : p.halo_in_r + xslot + (lane - (32 - HL)) * VP;
      else if (need)
        s = edges + ((size_t)nbq * 4 + (band & 3)) * 2 * HB + (lhalo ? HB + lane * VP : (lane - (32 - HL)) * VP);
      uint64_t pr[VP];
      bool ok = true;
      if (need) {
#pragma unroll
        for (int v = 0; v < VP; v += 2) {
          if (xin) cb_ld_pair2_sys(s + v, pr[v], pr[v + 1]);
          else cb_ld_pair2(s + v, pr[v], pr[v + 1]);
        }
#pragma unroll
        for (int v = 0; v < VP; ++v) ok = ok && ((uint32_t)(pr[v] >> 32) == tag);
      }
      if (!__all_sync(0xffffffffu, ok)) {
        Backoff bo;
        int spins = 0;
        while (true) {
          if (!ok) {
            ok = true;
#pragma unroll
            for (int v = 0; v < VP; v += 2) {
              if (xin) cb_ld_pair2_sys(s + v, pr[v], pr[v + 1]);
              else cb_ld_pair2(s + v, pr[v], pr[v + 1]);
            }
#pragma unroll
            for (int v = 0; v < VP; ++v) ok = ok && ((uint32_t)(pr[v] >> 32) == tag);
          }
          if (__all_sync(0xffffffffu, ok)) break;
          // busy-poll first (the neighbour is normally within an L2 round trip), then back off
          if (++spins > 64 && !bo.tick(ctl, p.timeout_ns)) return;
        }
      }
      if (need) {
#pragma unroll
        for (int v = 0; v < VP; ++v) cur[v] = (T)(uint32_t)pr[v];
      }
      if (trc) p.trace[2 * (r0 / HB) + 1] = (uint64_t)(clock64() - tb0);
    }
    if constexpr (MODE == 0) cp_async_wait_group<0>();

    // ---- outputs of the last row
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
      unsigned* rowmin_done = &ctl->pad[0];
      T* rowmins = reinterpret_cast<T*>(p.prog);
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, off));
      if (lane == 0) {
        rowmins[q] = mn;
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

// ---------------------------------------------------------------------------------------------
// Compiled geometries: variant id -> (VP, HB, D); BW = 32*VP - 2*HB own columns per warp.
// ---------------------------------------------------------------------------------------------
// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link needed).
static PFN_cuTensorMapEncodeTiled_v12000 cb_encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (fn == nullptr) {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
  }
  return fn;
}

template <class F, int VP, int HB, int D, int MODE = 0>
static cudaError_t cb_launch(const FillParams& p, int nw, bool query, int* out, cudaStream_t s) {
  const size_t smem = (size_t)nw * D * 32 * VP * sizeof(typename F::GridT) + (MODE ? (size_t)nw * D * 8 : 0);
  auto kt = prevrow_cb_kernel<F, VP, HB, D, true, MODE>;
  auto kf = prevrow_cb_kernel<F, VP, HB, D, false, MODE>;
  cudaError_t e = cudaFuncSetAttribute(kt, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  auto k = p.table != nullptr ? kt : kf;
  if (query) {   // out = {own columns per warp, co-resident CTAs per SM}
    int occ = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, nw * 32, smem);
    out[0] = 32 * VP - 2 * HB;
    out[1] = occ;
    if (MODE == 2 && cb_encode_fn() == nullptr) out[1] = 0;   // no tensor-map encoder: not usable
    return e;
  }
  CUtensorMap tm;
  memset(&tm, 0, sizeof(tm));
  if (MODE == 2) {   // the cost grid as a 2-D int32 tensor, box = kCbRG rows x the warp's window
    PFN_cuTensorMapEncodeTiled_v12000 enc = cb_encode_fn();
    if (enc == nullptr) return cudaErrorNotSupported;
    const cuuint64_t dims[2] = {(cuuint64_t)p.cols, (cuuint64_t)p.rows};
    const cuuint64_t strides[1] = {(cuuint64_t)p.grid_pitch * sizeof(typename F::GridT)};
    const cuuint32_t box[2] = {(cuuint32_t)(32 * VP), (cuuint32_t)kCbRG};
    const cuuint32_t estr[2] = {1, 1};
    if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_INT32, 2, const_cast<void*>(p.grid), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return cudaErrorInvalidValue;
  }
  const int grid = (p.nblocks + nw - 1) / nw;
  FillParams pp = p;
  void* args[] = {&pp, &tm};
  return cudaLaunchCooperativeKernel((const void*)k, dim3(grid), dim3(nw * 32), args, smem, s);
}

template <class F>
static cudaError_t cb_dispatch(int variant, const FillParams& p, int nw, bool query, int* out, cudaStream_t s) {
  switch (variant) {
    case 0: return cb_launch<F, 8, 64, 48>(p, nw, query, out, s);   // BW 128
    case 5: return cb_launch<F, 4, 32, 64>(p, nw, query, out, s);   // BW 64
    case 13: return cb_launch<F, 2, 16, 64>(p, nw, query, out, s);      // BW 32, 8-byte segments, 1024 warps for C4
    case 17: return cb_launch<F, 6, 48, 48>(p, nw, query, out, s);      // BW 96, exchange every 48 rows
    default: return cudaErrorInvalidValue;
  }
}

// query = true: out[0] = own columns per warp (BW), out[1] = co-resident CTAs per SM.
cudaError_t launch_prevrow_cb(int func, int variant, const FillParams& p, int nw, bool query, int* out,
                              cudaStream_t s) {
  switch (func) {
    case 3: return cb_dispatch<CellMinPath3>(variant, p, nw, query, out, s);
    case 4: return cb_dispatch<CellDiagMaxPlus>(variant, p, nw, query, out, s);
    case 5: return cb_dispatch<CellMin2Plus>(variant, p, nw, query, out, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace lddp
