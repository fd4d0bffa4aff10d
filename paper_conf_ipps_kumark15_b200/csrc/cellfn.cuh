// cellfn.cuh -- the compiled-in cell functions f of the LDDP-Plus recurrence
//     table[i][j] = f(L, UL, U, UR)          [L30 §I], [L94 §II], RS(i,j) [L90]
// and the initialisation each f implies [L300-L313].  Every functor declares its contributing
// set (kMask, Table I [L124-L142]) and supplies:
//   top(gc)   value of the row above the f-region (table row 0) at global column gc in [-1, n]
//   left(i)   value of the column left of the f-region at row i   (table column 0)
//   right(i)  value right of the last column (only read through UR)
//   row_ctx / col_ctx / load   per-row, per-column and per-cell inputs
//   f(...)    the cell update; writes the table-output element into `o`
// Readings of the paper (R1..R9) are listed in DESIGN.md §3.
#pragma once
#include <cstdint>
#include <climits>
#include "params.h"

namespace lddp {

enum : uint32_t { NB_L = 1u, NB_UL = 2u, NB_U = 4u, NB_UR = 8u };
enum ScoreKind { SCORE_NONE = 0, SCORE_LAST_CELL = 1, SCORE_ROW_MIN = 2 };

// ---------------------------------------------------------------------------------------- LCS
// [L88] Fig. 1(c) contributing set {L,UL,U}; textbook recurrence (reading R1) in the exact
// integer form max(U, L, UL + [a_i = b_j]) (equal to the textbook branch form because
// adjacent LCS cells differ by at most 1).
// Run-time 1 for integer adds the compiler must not fold into VIADD: VIADD issues on the ALU
// pipe together with ISETP / VIMNMX3, IMAD on the FMA pipe (balances the two pipes).
__device__ __forceinline__ int32_t imad_add1(int32_t x, int32_t one) {
  int32_t r;
  asm("mad.lo.s32 %0, %1, %2, %2;" : "=r"(r) : "r"(x), "r"(one));
  return r;
}

struct CellLCS {
  using T = int32_t;
  using RowCtx = int32_t;
  using ColCtx = int32_t;
  using GridT = int32_t;
  using OutT = int32_t;
  static constexpr uint32_t kMask = NB_L | NB_UL | NB_U;
  static constexpr bool kGridIn = false;
  static constexpr int kScore = SCORE_LAST_CELL;
  __device__ static RowCtx row_ctx(const FillParams& p, int64_t i) {
    return static_cast<const uint8_t*>(p.a)[i];
  }
  __device__ static ColCtx col_ctx(const FillParams& p, int gc) {
    return static_cast<const uint8_t*>(p.b)[gc];
  }
  __device__ static T top(const FillParams&, int) { return 0; }
  __device__ static T left(const FillParams&, int64_t) { return 0; }
  __device__ static T right(const FillParams&, int64_t) { return 0; }
  // virtual rows above row 0 (adiag.cuh): a character that matches nothing, boundary 0 -- f
  // then regenerates the all-zero row 0 of the table by itself
  __device__ static RowCtx vrow() { return -1; }
  __device__ static T vbig() { return 0; }
  __device__ static GridT load(const FillParams&, int64_t, int) { return 0; }
  __device__ static void prefetch_l1(const FillParams&, int64_t, int) {}
  __device__ __forceinline__ static T f(T L, T UL, T U, T, RowCtx a, ColCtx b, GridT, int64_t,
                                        int, int, OutT& o) {
    T v = max(max(U, L), UL + (a == b ? 1 : 0));
    o = v;
    return v;
  }
  // The same cell for adiag.cuh, given eq = [a_i = b_j] from the per-lane match table (one
  // shared-memory lookup + one R2P per step instead of one ISETP per cell): the +1 is a
  // predicated IMAD on the FMA pipe (`one` is a run-time 1), the 3-way max one VIMNMX3.
  static constexpr bool kMatchCells = true;
  __device__ __forceinline__ static T fad(T, T, T, RowCtx, ColCtx, int32_t) { return T(0); }
  __device__ __forceinline__ static T fadm(T L, T UL, T U, bool eq, int32_t one) {
    const T ulp = imad_add1(UL, one);
    const T t = eq ? ulp : UL;
    return max(max(U, L), t);
  }
};

// -------------------------------------------------------------------------------- Levenshtein
// [L319-L329] §VI.A with the restored min (reading R7): boundary max(i,j); equal characters
// copy UL, else 1 + min(U, L, UL).
struct CellLev {
  using T = int32_t;
  using RowCtx = int32_t;
  using ColCtx = int32_t;
  using GridT = int32_t;
  using OutT = int32_t;
  static constexpr uint32_t kMask = NB_L | NB_UL | NB_U;
  static constexpr bool kGridIn = false;
  static constexpr int kScore = SCORE_LAST_CELL;
  __device__ static RowCtx row_ctx(const FillParams& p, int64_t i) {
    return static_cast<const uint8_t*>(p.a)[i];
  }
  __device__ static ColCtx col_ctx(const FillParams& p, int gc) {
    return static_cast<const uint8_t*>(p.b)[gc];
  }
  __device__ static T top(const FillParams&, int gc) { return gc + 1; }           // f(0, gc+1)
  __device__ static T left(const FillParams&, int64_t i) { return (T)(i + 1); }   // f(i+1, 0)
  __device__ static T right(const FillParams&, int64_t) { return 0; }
  // virtual rows (adiag.cuh): never-matching character, boundary 2^30 above row -1, so that
  // row -1 = 1 + L regenerates f(0, j) = j (values stay >= 2^30 above it)
  __device__ static RowCtx vrow() { return -1; }
  __device__ static T vbig() { return 1 << 30; }
  __device__ static GridT load(const FillParams&, int64_t, int) { return 0; }
  __device__ static void prefetch_l1(const FillParams&, int64_t, int) {}
  __device__ __forceinline__ static T f(T L, T UL, T U, T, RowCtx a, ColCtx b, GridT, int64_t,
                                        int, int, OutT& o) {
    T v = (a == b) ? UL : 1 + min(min(U, L), UL);
    o = v;
    return v;
  }
  // adiag.cuh form (eq from the match table): the textbook min(U+1, L+1, UL+[a!=b]), equal in
  // integers to the form above because adjacent edit-distance cells differ by at most 1 (and
  // in the virtual rows above row 0 every value is >= 2^30, so row -1 is still L+1).
  static constexpr bool kMatchCells = true;
  __device__ __forceinline__ static T fad(T, T, T, RowCtx, ColCtx, int32_t) { return T(0); }
  __device__ __forceinline__ static T fadm(T L, T UL, T U, bool eq, int32_t one) {
    const T t = eq ? UL : imad_add1(UL, one);
    return min(min(imad_add1(U, one), imad_add1(L, one)), t);
  }
};

// ---------------------------------------------------------------------------------------- DTW
// [L26] + reading R2: D[0][0] = 0, D[i][0] = D[0][j] = +inf; binary32
// D = |x_i - y_j| + min(min(U, L), UL) -- the oracle's exact operation sequence (one rounded
// subtraction, exact mins, one rounded add), so the result is bit-identical.
struct CellDTW {
  using T = float;
  using RowCtx = float;
  using ColCtx = float;
  using GridT = float;
  using OutT = float;
  static constexpr uint32_t kMask = NB_L | NB_UL | NB_U;
  static constexpr bool kGridIn = false;
  static constexpr int kScore = SCORE_LAST_CELL;
  __device__ static RowCtx row_ctx(const FillParams& p, int64_t i) {
    return static_cast<const float*>(p.a)[i];
  }
  __device__ static ColCtx col_ctx(const FillParams& p, int gc) {
    return static_cast<const float*>(p.b)[gc];
  }
  __device__ static T top(const FillParams&, int gc) { return gc == -1 ? 0.0f : __int_as_float(0x7f800000); }
  __device__ static T left(const FillParams&, int64_t) { return __int_as_float(0x7f800000); }
  __device__ static T right(const FillParams&, int64_t) { return __int_as_float(0x7f800000); }
  // virtual rows (adiag.cuh): x = +inf makes every cost +inf, so row -1 = +inf for j >= 0
  __device__ static RowCtx vrow() { return __int_as_float(0x7f800000); }
  __device__ static T vbig() { return __int_as_float(0x7f800000); }
  __device__ static GridT load(const FillParams&, int64_t, int) { return 0.0f; }
  __device__ static void prefetch_l1(const FillParams&, int64_t, int) {}
  __device__ __forceinline__ static T f(T L, T UL, T U, T, RowCtx x, ColCtx y, GridT, int64_t,
                                        int, int, OutT& o) {
    float cost = fabsf(__fsub_rn(x, y));
    float v = __fadd_rn(cost, fminf(fminf(U, L), UL));
    o = v;
    return v;
  }
  static constexpr bool kMatchCells = false;
  __device__ __forceinline__ static T fadm(T, T, T, bool, int32_t) { return T(0); }
  __device__ __forceinline__ static T fad(T L, T UL, T U, RowCtx x, ColCtx y, int32_t) {
    return __fadd_rn(fabsf(__fsub_rn(x, y)), fminf(fminf(U, L), UL));
  }
};

// ------------------------------------------------------------------------- Floyd-Steinberg
// [L341-L344] §VI.B.  The carried cell value is the diffusion error e of the pixel.  Pull form
// of the raster push form: the four contributions reach pixel (i,j) in raster order UL, U, UR,
// L, so v = (((in + e_UL*1/16) + e_U*5/16) + e_UR*3/16) + e_L*7/16 with every product and sum
// rounded separately (__fmul_rn / __fadd_rn are never contracted to FFMA) -- bit-identical to
// the oracle.  Absent neighbours carry e = 0 (+0.0 adds are exact).  Threshold 128, ties to
// 255 (reading R3); e = v - out (reading R4).
struct CellFS {
  using T = float;
  using RowCtx = int32_t;
  using ColCtx = int32_t;
  using GridT = float;
  using OutT = uint8_t;
  static constexpr uint32_t kMask = NB_L | NB_UL | NB_U | NB_UR;
  static constexpr bool kGridIn = true;
  static constexpr bool kByteIO = true;   // uint8 grid in, uint8 table out (word-vectorisable)
  static constexpr int kScore = SCORE_NONE;
  __device__ static RowCtx row_ctx(const FillParams&, int64_t) { return 0; }
  __device__ static ColCtx col_ctx(const FillParams&, int) { return 0; }
  __device__ static GridT from_byte(uint32_t b) { return (float)b; }
  __device__ static T top(const FillParams&, int) { return 0.0f; }
  __device__ static T left(const FillParams&, int64_t) { return 0.0f; }
  __device__ static T right(const FillParams&, int64_t) { return 0.0f; }
  __device__ static GridT load(const FillParams& p, int64_t i, int c) {
    return (float)__ldg(static_cast<const uint8_t*>(p.grid) + i * p.grid_pitch + c);
  }
  __device__ static void prefetch_l1(const FillParams& p, int64_t i, int c) {
    asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(static_cast<const uint8_t*>(p.grid) + i * p.grid_pitch + c));
  }
  __device__ __forceinline__ static T f(T L, T UL, T U, T UR, RowCtx, ColCtx, GridT in, int64_t,
                                        int, int, OutT& o) {
    float v = __fadd_rn(in, __fmul_rn(UL, 0.0625f));
    v = __fadd_rn(v, __fmul_rn(U, 0.3125f));
    v = __fadd_rn(v, __fmul_rn(UR, 0.1875f));
    v = __fadd_rn(v, __fmul_rn(L, 0.4375f));
    // threshold as a register mask (set.ge.u32.f32) rather than a branch-like select of two
    // results: m = v >= 128 ? ~0 : 0; e = v - (m & bits(255.0f)), exactly the oracle's v - 255 or
    // v - (+0) = v.  (An integer-compare formulation on the bits measured slower: C3 1.57 -> 1.62 ms.)
    uint32_t m;
    asm("set.ge.u32.f32 %0, %1, 128.0;" : "=r"(m) : "f"(v));
    o = (uint8_t)(m & 255u);
    return __fsub_rn(v, __uint_as_float(m & 0x437F0000u));
  }
};

// ------------------------------------------------------------------------------ MIN_PATH3
// [L350-L367] §VI.C checkerboard, reading R6: f[0][j] = c[0][j]; f = c + min over the in-range
// {UL, U, UR}.  Out-of-range neighbours are INT_MAX, used only as min operands.  The row above
// row 0 is 0 inside the grid, so f[0][j] = c[0][j] + 0.
struct CellMinPath3 {
  using T = int32_t;
  using RowCtx = int32_t;
  using ColCtx = int32_t;
  using GridT = int32_t;
  using OutT = int32_t;
  static constexpr uint32_t kMask = NB_UL | NB_U | NB_UR;
  static constexpr bool kGridIn = true;
  static constexpr int kScore = SCORE_ROW_MIN;
  __device__ static RowCtx row_ctx(const FillParams&, int64_t) { return 0; }
  __device__ static ColCtx col_ctx(const FillParams&, int) { return 0; }
  __device__ static T top(const FillParams& p, int gc) {
    return (gc >= 0 && gc < p.cols_total) ? 0 : INT_MAX;
  }
  __device__ static T left(const FillParams&, int64_t) { return INT_MAX; }
  __device__ static T right(const FillParams&, int64_t) { return INT_MAX; }
  __device__ static GridT load(const FillParams& p, int64_t i, int c) {
    return __ldg(static_cast<const int32_t*>(p.grid) + i * p.grid_pitch + c);
  }
  __device__ static void prefetch_l1(const FillParams& p, int64_t i, int c) {
    asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(static_cast<const int32_t*>(p.grid) + i * p.grid_pitch + c));
  }
  __device__ __forceinline__ static T f(T, T UL, T U, T UR, RowCtx, ColCtx, GridT g, int64_t,
                                        int, int, OutT& o) {
    T v = g + __vimin3_s32(UL, U, UR);   // VIMNMX3
    o = v;
    return v;
  }
};

// ------------------------------------------------------------------------------ MIN2_PLUS
// [L298] §V.B Horizontal case-1 synthetic f = min(UL, U) + c; row 0 = init (reading R8);
// UL at j = 0 is INT_MAX (excluded).
struct CellMin2Plus {
  using T = int32_t;
  using RowCtx = int32_t;
  using ColCtx = int32_t;
  using GridT = int32_t;
  using OutT = int32_t;
  static constexpr uint32_t kMask = NB_UL | NB_U;
  static constexpr bool kGridIn = true;
  static constexpr int kScore = SCORE_ROW_MIN;
  __device__ static RowCtx row_ctx(const FillParams&, int64_t) { return 0; }
  __device__ static ColCtx col_ctx(const FillParams&, int) { return 0; }
  __device__ static T top(const FillParams&, int) { return 0; }
  __device__ static T left(const FillParams&, int64_t) { return INT_MAX; }
  __device__ static T right(const FillParams&, int64_t) { return INT_MAX; }
  __device__ static GridT load(const FillParams& p, int64_t i, int c) {
    return __ldg(static_cast<const int32_t*>(p.grid) + i * p.grid_pitch + c);
  }
  __device__ static void prefetch_l1(const FillParams& p, int64_t i, int c) {
    asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(static_cast<const int32_t*>(p.grid) + i * p.grid_pitch + c));
  }
  __device__ __forceinline__ static T f(T, T UL, T U, T, RowCtx, ColCtx, GridT g, int64_t i,
                                        int, int pc, OutT& o) {
    T v = (i == 0) ? g : min(UL, U) + pc;
    o = v;
    return v;
  }
};

// --------------------------------------------------------------------------- DIAG_MAXPLUS
// [L298] §V.B Inverted-L synthetic f = max(cell_{i,j}, f(i-1,j-1)) + c, cell = init (reading
// R9); row 0 and column 0 are init.
struct CellDiagMaxPlus {
  static constexpr bool kDirectGrid = true;   // invl.cuh streams the grid with a running pointer
  using T = int32_t;
  using RowCtx = int32_t;
  using ColCtx = int32_t;
  using GridT = int32_t;
  using OutT = int32_t;
  static constexpr uint32_t kMask = NB_UL;
  static constexpr bool kGridIn = true;
  static constexpr int kScore = SCORE_NONE;
  __device__ static RowCtx row_ctx(const FillParams&, int64_t) { return 0; }
  __device__ static ColCtx col_ctx(const FillParams&, int) { return 0; }
  __device__ static T top(const FillParams&, int) { return 0; }
  __device__ static T left(const FillParams&, int64_t) { return 0; }
  __device__ static T right(const FillParams&, int64_t) { return 0; }
  __device__ static GridT load(const FillParams& p, int64_t i, int c) {
    return __ldg(static_cast<const int32_t*>(p.grid) + i * p.grid_pitch + c);
  }
  __device__ static void prefetch_l1(const FillParams& p, int64_t i, int c) {
    asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(static_cast<const int32_t*>(p.grid) + i * p.grid_pitch + c));
  }
  __device__ __forceinline__ static T f(T, T UL, T, T, RowCtx, ColCtx, GridT g, int64_t i,
                                        int gc, int pc, OutT& o) {
    T v = (i == 0 || gc == 0) ? g : max(g, UL) + pc;
    o = v;
    return v;
  }
};

}  // namespace lddp
