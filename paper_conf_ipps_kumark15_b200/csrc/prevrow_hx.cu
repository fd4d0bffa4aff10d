// prevrow_hx.cu -- previous-row-only ("Horizontal", t = i) category: hierarchical-exchange
// column-block kernel, the default prev-row kernel on one GPU (C4, C7; SCORE / LAST_ROW and
// TABLE) [L180-L195], Fig. 2(b).  prevrow_cb.cu remains the multi-GPU / band_rows / unaligned-
// TABLE path.
//
// Why a second column-block kernel.  prevrow_cb exchanges every warp's trapezoid halos through
// L2 every HB = 32 rows; one store -> load visibility between SMs costs ~860 cycles
// (tools/micro/l2rt.cu), the exchange is two-way, so every band pays C_band + ~1500 cycles on
// the critical path: ~0.9 of C4's 2.0 ms.  Here:
//
//  * Two exchange levels (Table II case-2 two-way halo [L265-L274], [L193-L195], applied
//    hierarchically).  A CTA of NW warps (one per SM sub-partition) owns CW consecutive
//    columns.  Warps of a CTA exchange their inner halos (HBI columns) through shared memory
//    every HBI rows with one named barrier; only the CTA's two outer edges go through L2, every
//    HBO rows, with HBO-column outer halos carried by the CTA's edge warps.  The L2 round trip
//    is paid once per HBO rows instead of once per 32.  Default HBI 16, HBO 96: C4 1.54 ms.
//  * Optional lane ghosts (GH = 2, variant 0): every lane keeps GH copies of each neighbour
//    lane's edge columns, refreshed by SHFL every GH rows (garbage entering a lane window's edge
//    advances one column per row -- the trapezoid argument one level down); measured no faster
//    than GH = 1 (the default), kept compiled.
//  * A fully unrolled band: ring slots, LDS and LDGSTS destinations are immediates; one
//    IMAD.WIDE forms each row's copy address; cp.async.wait once per GH rows.
//  * Table edges: column 0's UL and column W-1's UR are forced to f's boundary value with one
//    LOP3 each in the (warp-uniform) EDGE body only, in every lane that holds those columns.
//  * TABLE (TB): every own in-table lane stores its 4 new values per row with one 16-byte store.
//
// Geometry: lane l of warp w holds the VP = 4 columns [s_w + 4l, s_w + 4l + 4) of the warp's
// window [s_w, s_w + 128); hl(w) = HBO for w = 0 else HBI columns of left halo, hr(w) likewise
// on the right; own(w) = 128 - hl(w) - hr(w).  Columns >= W and < 0 are computed as garbage and
// never read by an in-table cell (the edge fixes).
#include <climits>
#include <cstdint>
#include <cstring>

#include "cellfn.cuh"
#include "params.h"
#include "sync.cuh"

namespace lddp {

namespace hx {

constexpr int VP = 4;
constexpr int EXT = 32 * VP;

__device__ __forceinline__ void cp16(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void wait_group() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ int4 lds128(uint32_t a) {
  int4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts128(uint32_t a, int4 v) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
template <int NT>
__device__ __forceinline__ void bar_named() {
  asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory");
}
__device__ __forceinline__ void st_pair2(uint64_t* p, uint64_t a, uint64_t b) {
  asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void ld_pair2(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
// system scope: edge pairs exchanged with the neighbour GPUs' comm windows (lddp_fill_multi)
__device__ __forceinline__ void st_pair2_sys(uint64_t* p, uint64_t a, uint64_t b) {
  asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void ld_pair2_sys(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.sys.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ uint32_t opq(uint32_t x) {
  asm volatile("mov.b32 %0, %0;" : "+r"(x));
  return x;
}
template <class T>
__device__ __forceinline__ T fix(T x, uint32_t A, uint32_t O) {
  uint32_t u;
  memcpy(&u, &x, 4);
  u = (u & A) | O;
  memcpy(&x, &u, 4);
  return x;
}

template <int NW, int HBI, int HBO>
struct Geo {
  __host__ __device__ static constexpr int hl(int w) { return w == 0 ? HBO : HBI; }
  __host__ __device__ static constexpr int hr(int w) { return w == NW - 1 ? HBO : HBI; }
  __host__ __device__ static constexpr int own(int w) { return EXT - hl(w) - hr(w); }
  __host__ __device__ static constexpr int ownoff(int w) { return w == 0 ? 0 : ownoff(w - 1) + own(w - 1); }
  static constexpr int CW = ownoff(NW - 1) + own(NW - 1);
  __host__ __device__ static constexpr bool ok() {
    for (int w = 0; w < NW; ++w)
      if (own(w) < HBI || own(w) < 4) return false;
    return CW >= 2 * HBO && HBO % HBI == 0 && HBI % VP == 0;
  }
};

}  // namespace hx

// Per-lane state and the row loop of one warp.
template <class F, int GH, int D, bool TB = false>
struct HxLane {
  using T = typename F::T;
  using G = typename F::GridT;
  static constexpr int NX = hx::VP + 2 * GH;   // x[GH + v] = own column v; ghosts on both sides
  T x[NX];
  uint32_t lA, lO, rA, rO;   // table-edge masks (EDGE bodies): UL of column 0, UR of column W-1
  uint32_t ring0;            // shared address of this lane's segment in slot 0
  const char* gsrc;          // global address of this lane's segment in row 0 (or the grid base)
  uint32_t gsz;              // 16, or 0 (zero-fill: columns outside the table)
  uint32_t pitchb;           // row pitch in bytes
  int hlast;                 // last table row (copies clamp to it)
  int e0;                    // first column of this lane
  char* tptr;                // TB: &table[0][e0] (own in-table lanes), else nullptr
  uint32_t tpitchb;          // TB: table row pitch in bytes

  __device__ __forceinline__ void issue(int rr, uint32_t dst) const {
    const int rc = min(rr, hlast);
    const char* src = gsrc + (uint64_t)(uint32_t)rc * pitchb;
    hx::cp16(dst, src, gsz);
    hx::commit();
  }

  // One period of GH rows starting at row r (slot sl = r mod D).  NR < GH only in the last band.
  template <bool EDGE>
  __device__ __forceinline__ void period(const FillParams& p, int r, int sl, int nr) {
    constexpr int VP = hx::VP;
    constexpr int RB = hx::EXT * 4;   // ring row bytes
    // costs of the period's rows (all landed: wait_group at the caller)
    G g[GH][VP];
#pragma unroll
    for (int t = 0; t < GH; ++t) {
      const int4 v = hx::lds128(ring0 + (uint32_t)((sl + t) * RB));
      g[t][0] = v.x; g[t][1] = v.y; g[t][2] = v.z; g[t][3] = v.w;
    }
    // ghost costs of row t < GH - 1 (columns e0 - 1 - ... and e0 + VP + ...): neighbour lanes' costs
    G gl[GH > 1 ? GH - 1 : 1][GH > 1 ? GH - 1 : 1], gr[GH > 1 ? GH - 1 : 1][GH > 1 ? GH - 1 : 1];
#pragma unroll
    for (int t = 0; t + 1 < GH; ++t) {
#pragma unroll
      for (int k = 0; k < GH - 1 - t; ++k) {
        gl[t][k] = __shfl_up_sync(0xffffffffu, g[t][VP - 1 - k], 1);   // column e0 - 1 - k
        gr[t][k] = __shfl_down_sync(0xffffffffu, g[t][k], 1);         // column e0 + VP + k
      }
    }
    // ghost refresh: x[GH-1-k] = lane-1's own column VP-1-k, x[GH+VP+k] = lane+1's own column k
#pragma unroll
    for (int k = 0; k < GH; ++k) {
      x[GH - 1 - k] = __shfl_up_sync(0xffffffffu, x[GH + VP - 1 - k], 1);
      x[GH + VP + k] = __shfl_down_sync(0xffffffffu, x[GH + k], 1);
    }
#pragma unroll
    for (int t = 0; t < GH; ++t) {
      if (t < nr) {
        if (EDGE) {
          x[GH - 1] = hx::fix(x[GH - 1], lA, lO);
          x[GH + VP] = hx::fix(x[GH + VP], rA, rO);
        }
        T y[NX];
        // row t updates x[1 + t .. NX - 2 - t]
#pragma unroll
        for (int j = 1 + t; j <= NX - 2 - t; ++j) {
          const int c = j - GH;   // column offset from the lane's first own column
          G gc;
          if (c >= 0 && c < VP) gc = g[t][c];
          else if (c < 0) gc = gl[t][-1 - c];
          else gc = gr[t][c - VP];
          typename F::OutT o;
          y[j] = F::f(x[j], x[j - 1], x[j], x[j + 1], typename F::RowCtx(0), typename F::ColCtx(0), gc,
                      (int64_t)(r + t), p.col0 + e0 + c, p.param_c, o);
        }
#pragma unroll
        for (int j = 1 + t; j <= NX - 2 - t; ++j) x[j] = y[j];
        if constexpr (TB) {   // TABLE: this row's own columns, one 16-byte store per lane
          if (tptr != nullptr) {
            char* d = tptr + (uint64_t)(uint32_t)(r + t) * tpitchb;
            *reinterpret_cast<int4*>(d) = make_int4(x[GH], x[GH + 1], x[GH + 2], x[GH + 3]);
          }
        }
      }
    }
  }
};

// One band of HBI rows (FULL) or the last rows (r0 .. H-1, all already in the ring).
template <class F, int GH, int D, bool TB, int HBI, bool EDGE, bool FULL>
__device__ __forceinline__ void hx_band(HxLane<F, GH, D, TB>& st, const FillParams& p, int r0, int H) {
  constexpr int RB = hx::EXT * 4;
  if constexpr (FULL) {
    const int sl0 = r0 % D;
    // HBI / GH periods; after each, copies of rows r + t + D - 1 go into the slots of rows r + t - 1
#pragma unroll
    for (int pt = 0; pt < HBI / GH; ++pt) {
      hx::wait_group<D - 1 - GH>();
      const int r = r0 + pt * GH;
      st.template period<EDGE>(p, r, sl0 + pt * GH, GH);
#pragma unroll
      for (int t = 0; t < GH; ++t) {
        const int s = sl0 + pt * GH + t - 1;   // -1: the ring's last slot
        st.issue(r + t + D - 1, st.ring0 + (uint32_t)((s < 0 ? s + D : s) * RB));
      }
    }
  } else {
    hx::wait_group<0>();
#pragma unroll 1
    for (int r = r0; r < H; r += GH) st.template period<EDGE>(p, r, r % D, H - r);
  }
}

template <class F, int NW, int HBI, int HBO, int D, int GH, bool TB, bool XR>
__global__ void __launch_bounds__(NW * 32, 1) prevrow_hx_kernel(const FillParams p) {
  using Geo = hx::Geo<NW, HBI, HBO>;
  static_assert(Geo::ok(), "hierarchical-exchange geometry");
  static_assert(D % HBI == 0 && HBI % GH == 0 && D > HBI + GH, "ring of whole bands");
  static_assert(!(F::kMask & NB_L), "prev-row category: f must not read L");
  using T = typename F::T;
  using L = HxLane<F, GH, D, TB>;
  constexpr int VP = hx::VP, EXT = hx::EXT, RB = EXT * 4;
  constexpr int CW = Geo::CW;

  extern __shared__ __align__(128) unsigned char hx_smem[];
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  const int c = blockIdx.x;
  const int nc = gridDim.x;
  const int W = p.cols;
  const int H = (int)p.rows;
  Control* ctl = static_cast<Control*>(p.ctl);

  int hl = HBI, ownw = 0, ownoff = 0;
#pragma unroll
  for (int v = 0; v < NW; ++v)
    if (v == w) { hl = Geo::hl(v); ownw = Geo::own(v); ownoff = Geo::ownoff(v); }
  const int hr = EXT - hl - ownw;
  const int A = c * CW;                  // first own column of the CTA
  const int sw = A + ownoff - hl;        // warp window start
  const int e0 = sw + lane * VP;         // first column of this lane
  const bool lhalo = lane * VP < hl, rhalo = lane * VP >= EXT - hr;
  const bool own = !lhalo && !rhalo;

  // shared memory: [16 B pad][NW x D ring rows][16 B pad][2 x exchange row of NW*EXT ints][reduction]
  const uint32_t sbase = smem_u32(hx_smem);
  L st;
  st.ring0 = sbase + 16 + (uint32_t)(w * D * RB + lane * 16);
  const uint32_t xs0 = sbase + 32 + (uint32_t)(NW * D * RB);
  const int xidx = e0 - (A - HBO);       // index in the CTA's extended window
  // local columns: [0, W) this rank's strip (outputs); [clo, chi) the whole table (costs: a
  // multi-GPU rank's halos read its neighbours' columns of the grid).  W % 4 == 0 and the strip
  // starts on a multiple of 4: a lane's 4 columns are all in or all out.
  // (XR: a multi-GPU rank's fill; the single-GPU instantiation keeps the window code out)
  const int clo = XR ? -p.col0 : 0, chi = XR ? p.cols_total - p.col0 : W;
  const bool in = e0 >= 0 && e0 < W;
  const bool gin = e0 >= clo && e0 < chi;
  st.gsz = hx::opq(gin ? 16u : 0u);
  st.gsrc = static_cast<const char*>(p.grid) + (gin ? (int64_t)e0 * 4 : 0);
  st.pitchb = (uint32_t)(p.grid_pitch * 4);
  st.hlast = H - 1;
  st.e0 = e0;
  st.tptr = (TB && own && in) ? static_cast<char*>(p.table) + (int64_t)e0 * 4 : nullptr;
  st.tpitchb = (uint32_t)(p.table_pitch * 4);

  // table-edge masks: every lane holding column 0 (v = 0) forces its UL, every lane holding column
  // W-1 (v = 3) its UR, to f's boundary values
  {
    const T lb = F::left(p, 0), rb = F::right(p, 0);
    uint32_t lbits, rbits;
    memcpy(&lbits, &lb, 4);
    memcpy(&rbits, &rb, 4);
    st.lA = hx::opq(e0 == clo ? 0u : ~0u);
    st.lO = hx::opq(e0 == clo ? lbits : 0u);
    st.rA = hx::opq(e0 == chi - VP ? 0u : ~0u);
    st.rO = hx::opq(e0 == chi - VP ? rbits : 0u);
  }
  const bool edge = __any_sync(0xffffffffu, e0 == clo || e0 == chi - VP);

  // row -1 (virtual): f's top initialisation (out-of-table columns: garbage, never read)
#pragma unroll
  for (int v = 0; v < VP; ++v) st.x[GH + v] = F::top(p, p.col0 + e0 + v);

  // prologue: rows 0 .. D-2 into slots 0 .. D-2
#pragma unroll 1
  for (int k = 0; k < D - 1; ++k) st.issue(k, st.ring0 + (uint32_t)(k * RB));

  // outer-edge pairs in global memory: [CTA][4 slots][2 sides][HBO] (value, tag)
  uint64_t* edges = reinterpret_cast<uint64_t*>(p.bnd);
  // multi-GPU (lddp_fill_multi): CTA 0's left and the last CTA's right outer edges go to / come
  // from the neighbour ranks' comm windows ([8 slots: fill parity x outer band mod 4][HBO] pairs
  // per side, system scope); the strip partition is CTA-aligned, so the rank's strip edges are
  // CTA edges.  Tags carry the rank-consistent fill count (bit 31 set).
  constexpr bool xrank = XR;
  const uint32_t tag0 = xrank ? (0x80000000u | (uint32_t)(p.wepoch & 0x7FFu) << 20) : (uint32_t)(p.epoch & 0x7FFu) << 20;
  // One-way f's (contributing set without UR: MIN2_PLUS, DIAG_MAXPLUS -- Table II case 1, one-way
  // transfer [L265-L274]): own columns depend only on columns to their left, so a CTA waits for
  // its left neighbour's edge and never for its right one -- the CTAs form a pipeline instead of
  // a lock-step chain.  With no back-pressure a producer may run any number of outer bands
  // ahead, so (one GPU) every outer band has its own slot: edges[CTA][NOB][HBO], never reused
  // within a fill (the tags tell fills apart).
  constexpr bool kOneWayF = !(F::kMask & NB_UR);
  const bool oneway = kOneWayF && !xrank;
  const int NOB = (H + HBO - 1) / HBO;
  const bool pub_l = own && e0 >= A && e0 < A + HBO && !oneway;    // CTA c-1 reads these
  const bool pub_r = own && e0 >= A + CW - HBO && e0 < A + CW;     // CTA c+1 reads these
  const bool xin = XR && ((w == 0 && lhalo && c == 0 && p.halo_in_l != nullptr) ||
                          (w == NW - 1 && rhalo && c + 1 == nc && p.halo_in_r != nullptr));
  const bool get_l = w == 0 && lhalo && (c > 0 || (XR && p.halo_in_l != nullptr));
  const bool get_r = w == NW - 1 && rhalo && (c + 1 < nc || (XR && p.halo_in_r != nullptr)) && !oneway;
  uint64_t* const xout = !XR ? nullptr
                         : (pub_l && c == 0 && p.halo_out_l != nullptr) ? p.halo_out_l + (e0 - A)
                         : ((pub_r && c + 1 == nc && p.halo_out_r != nullptr) ? p.halo_out_r + (e0 - (A + CW - HBO))
                                                                               : nullptr);
  const bool pub = pub_l || pub_r, get = get_l || get_r;
  const bool ihalo = !own && !((w == 0 && lhalo) || (w == NW - 1 && rhalo));   // inner halo lane
  // this lane's pair addresses in slot 0 (slot s adds s * 2 * HBO): own edge columns it publishes,
  // neighbour columns it polls
  uint64_t* const pubp =
      oneway ? edges + (size_t)c * NOB * HBO + (e0 - (A + CW - HBO))
             : edges + ((size_t)c * 8 + (pub_l ? 0 : 1)) * HBO + (pub_l ? e0 - A : e0 - (A + CW - HBO));
  const uint64_t* const getp =
      xin ? (get_l ? p.halo_in_l + (e0 - (A - HBO)) : p.halo_in_r + (e0 - (A + CW)))
          : (oneway ? edges + (size_t)(c - 1) * NOB * HBO + (e0 - (A - HBO))
                    : (get_l ? edges + ((size_t)(c - 1) * 8 + 1) * HBO + (e0 - (A - HBO))
                             : edges + ((size_t)(c + 1) * 8 + 0) * HBO + (e0 - (A + CW))));
  const size_t xpar_slot = (size_t)(p.wepoch & 1) * 4;   // window slot base of this fill
  const uint32_t xsa = xs0 + (uint32_t)(xidx * 4);
  uint32_t xpar = 0;
  int kin = 0, ob = 0;   // inner band within the outer band, outer band
  bool aborted = false;

  // development trace (LDDP_TRACE, tools/hx_trace.py): CTA trace_chunks, lane 0 of every warp,
  // per inner band: cycles to the end of the band's rows and to the end of its exchange
  // (compiled in only with -DLDDP_HX_TRACE: the per-band checks cost ~10 % of C4)
#ifdef LDDP_HX_TRACE
  const bool trc = p.trace != nullptr && c == p.trace_chunks && lane == 0;
  const bool dbg_no_outer = (p.debug & 1) != 0, dbg_no_inner = (p.debug & 2) != 0;   // timing only
#else
  constexpr bool trc = false, dbg_no_outer = false, dbg_no_inner = false;
#endif
#pragma unroll 1
  for (int r0 = 0; r0 < H; r0 += HBI) {
    const long long tb0 = trc ? clock64() : 0;
    if (r0 + HBI <= H) {
      if (edge) hx_band<F, GH, D, TB, HBI, true, true>(st, p, r0, H);
      else hx_band<F, GH, D, TB, HBI, false, true>(st, p, r0, H);
    } else {
      if (edge) hx_band<F, GH, D, TB, HBI, true, false>(st, p, r0, H);
      else hx_band<F, GH, D, TB, HBI, false, false>(st, p, r0, H);
    }
    if (trc && r0 / HBI < 4096) p.trace[((r0 / HBI) * NW + w) * 2] = (uint64_t)(clock64() - tb0);
    if (r0 + HBI >= H) break;

    // ---- inner band boundary: own columns -> shared exchange row, halos <- neighbours
    const uint32_t xs = xsa + xpar;
    xpar ^= (uint32_t)(NW * EXT * 4);
    if (own) hx::sts128(xs, make_int4(st.x[GH], st.x[GH + 1], st.x[GH + 2], st.x[GH + 3]));
    const bool outer = kin == HBO / HBI - 1;   // an outer band (HBO rows) ends here
    kin = outer ? 0 : kin + 1;
    const uint32_t tag = tag0 | (((uint32_t)ob + 1u) & 0xFFFFFu);
    const size_t soff = oneway ? (size_t)ob * HBO : (size_t)(ob & 3) * 2 * HBO;   // this band's slot
    if (outer && pub) {
      uint64_t* d = pubp + soff;
      const uint64_t th = (uint64_t)tag << 32;
      hx::st_pair2(d, th | (uint32_t)st.x[GH], th | (uint32_t)st.x[GH + 1]);
      hx::st_pair2(d + 2, th | (uint32_t)st.x[GH + 2], th | (uint32_t)st.x[GH + 3]);
      if (XR && xout != nullptr) {   // the strip's outer edge -> the neighbour rank's window
        uint64_t* x = xout + (xpar_slot + (ob & 3)) * HBO;
        hx::st_pair2_sys(x, th | (uint32_t)st.x[GH], th | (uint32_t)st.x[GH + 1]);
        hx::st_pair2_sys(x + 2, th | (uint32_t)st.x[GH + 2], th | (uint32_t)st.x[GH + 3]);
      }
    }
    if (!dbg_no_inner) {
      hx::bar_named<NW * 32>();
      if (ihalo) {
        const int4 v = hx::lds128(xs);
        st.x[GH] = v.x; st.x[GH + 1] = v.y; st.x[GH + 2] = v.z; st.x[GH + 3] = v.w;
      }
    }
    if (outer && (w == 0 || w == NW - 1) && !dbg_no_outer) {
      const uint64_t* s = getp + (xin ? (xpar_slot + (ob & 3)) * HBO : soff);
      const bool need = get && !aborted;
      uint64_t pr[VP];
      bool ok = true;
      if (need) {
        if (XR && xin) {
          hx::ld_pair2_sys(s, pr[0], pr[1]);
          hx::ld_pair2_sys(s + 2, pr[2], pr[3]);
        } else {
          hx::ld_pair2(s, pr[0], pr[1]);
          hx::ld_pair2(s + 2, pr[2], pr[3]);
        }
#pragma unroll
        for (int v = 0; v < VP; ++v) ok = ok && ((uint32_t)(pr[v] >> 32) == tag);
      }
      if (!__all_sync(0xffffffffu, ok)) {
        Backoff bo;
        int spins = 0;
        while (true) {
          if (!ok) {
            if (XR && xin) {
              hx::ld_pair2_sys(s, pr[0], pr[1]);
              hx::ld_pair2_sys(s + 2, pr[2], pr[3]);
            } else {
              hx::ld_pair2(s, pr[0], pr[1]);
              hx::ld_pair2(s + 2, pr[2], pr[3]);
            }
            ok = true;
#pragma unroll
            for (int v = 0; v < VP; ++v) ok = ok && ((uint32_t)(pr[v] >> 32) == tag);
          }
          if (__all_sync(0xffffffffu, ok)) break;
          // busy-poll first (the neighbour is normally within an L2 round trip), then back off;
          // on abort / timeout keep computing (garbage) so the CTA's barriers still complete
          if (++spins > 64 && !bo.tick(ctl, p.timeout_ns)) {
            aborted = true;
            ok = true;
          }
        }
        aborted = __any_sync(0xffffffffu, aborted);
      }
      if (need && !aborted) {
#pragma unroll
        for (int v = 0; v < VP; ++v) st.x[GH + v] = (T)(uint32_t)pr[v];
      }
    }
    if (outer) ++ob;
    if (trc && r0 / HBI < 4096) p.trace[((r0 / HBI) * NW + w) * 2 + 1] = (uint64_t)(clock64() - tb0);
  }
  hx::wait_group<0>();

  // ---- outputs of the last row: last_row, and the row minimum (score) over all CTAs
  T mn = INT_MAX;
  if (own && in) {
#pragma unroll
    for (int v = 0; v < VP; ++v) {
      if (p.last_row != nullptr) static_cast<T*>(p.last_row)[e0 + v] = st.x[GH + v];
      mn = min(mn, st.x[GH + v]);
    }
  }
  if (F::kScore == SCORE_ROW_MIN && p.score != nullptr) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, off));
    T* red = reinterpret_cast<T*>(hx_smem + 48 + NW * D * RB + 2 * NW * EXT * 4);
    if (lane == 0) red[w] = mn;
    __syncthreads();
    if (threadIdx.x == 0) {
      for (int v = 1; v < NW; ++v) mn = min(mn, red[v]);
      unsigned* dn = &ctl->pad[0];
      T* mins = reinterpret_cast<T*>(p.prog);
      mins[c] = mn;
      __threadfence();
      const unsigned d = atomicAdd(dn, 1u);
      if (d == (unsigned)nc - 1) {
        __threadfence();
        T best = INT_MAX;
        for (int k = 0; k < nc; ++k) best = min(best, __ldcg(mins + k));
        *static_cast<T*>(p.score) = best;
        atomicExch(dn, 0u);
      }
    }
  }
}

// ---------------------------------------------------------------------------------------------
// Compiled geometries (variant id -> NW, HBI, HBO, D, GH); see DESIGN.md §5.2a.
// ---------------------------------------------------------------------------------------------
template <class F, int NW, int HBI, int HBO, int D, int GH>
static cudaError_t hx_launch(const FillParams& p, bool query, int* out, cudaStream_t s) {
  using Geo = hx::Geo<NW, HBI, HBO>;
  const size_t smem = 48 + (size_t)NW * D * hx::EXT * 4 + 2 * (size_t)NW * hx::EXT * 4 + 64;
  // TABLE fills: the TB instantiation (16-byte row stores; pitch and base checked by the caller);
  // multi-GPU rank fills: the XR instantiation (comm-window edges)
  const bool xr = p.halo_in_l != nullptr || p.halo_in_r != nullptr;
  decltype(&prevrow_hx_kernel<F, NW, HBI, HBO, D, GH, false, false>) ks[2][2] = {
      {prevrow_hx_kernel<F, NW, HBI, HBO, D, GH, false, false>, prevrow_hx_kernel<F, NW, HBI, HBO, D, GH, false, true>},
      {prevrow_hx_kernel<F, NW, HBI, HBO, D, GH, true, false>, prevrow_hx_kernel<F, NW, HBI, HBO, D, GH, true, true>}};
  auto k = ks[p.table != nullptr][xr];
  cudaError_t e = cudaSuccess;
  for (int a = 0; a < 2 && e == cudaSuccess; ++a)
    for (int b = 0; b < 2 && e == cudaSuccess; ++b)
      e = cudaFuncSetAttribute(ks[a][b], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (query) {   // out = {own columns per CTA, co-resident CTAs per SM, outer halo HBO}
    int occ = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, NW * 32, smem);
    out[0] = Geo::CW;
    out[1] = occ;
    out[2] = HBO;
    return e;
  }
  const int grid = (p.cols + Geo::CW - 1) / Geo::CW;
  FillParams pp = p;
  void* args[] = {&pp};
  return cudaLaunchCooperativeKernel((const void*)k, dim3(grid), dim3(NW * 32), args, smem, s);
}

template <class F>
static cudaError_t hx_dispatch(int variant, const FillParams& p, bool query, int* out, cudaStream_t s) {
  switch (variant) {
    // measured alternatives kept compiled; rejected ones are not built
    case 0: return hx_launch<F, 4, 16, 96, 64, 2>(p, query, out, s);   // lane ghosts (GH = 2)
    case 2: return hx_launch<F, 4, 16, 96, 64, 1>(p, query, out, s);   // default: CW 224, 147 CTAs for C4
    case 6: return hx_launch<F, 4, 16, 64, 64, 1>(p, query, out, s);   // HBO 64: CW 288
    case 8: return hx_launch<F, 4, 16, 96, 32, 1>(p, query, out, s);   // 32-row ring
    default: return cudaErrorInvalidValue;
  }
}

// query = true: out[0] = own columns per CTA, out[1] = co-resident CTAs per SM, out[2] = HBO.
cudaError_t launch_prevrow_hx(int func, int variant, const FillParams& p, bool query, int* out, cudaStream_t s) {
  switch (func) {
    case 3: return hx_dispatch<CellMinPath3>(variant, p, query, out, s);
    case 4: return hx_dispatch<CellDiagMaxPlus>(variant, p, query, out, s);
    case 5: return hx_dispatch<CellMin2Plus>(variant, p, query, out, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace lddp
