/*
 * lddp_user.cuh -- header-only fill for a USER-SUPPLIED cell function f (CUDA C++, sm_100a).
 *
 * "A user ... needs to supply only the problem dependent function f" [L45 §I], [L312 §V.C]: the
 * framework maps f's contributing set to a pattern [L113] (Table I [L124-L142]) and fills the
 * table in dependency order.  This header instantiates the library's generic category kernels
 * (the strip-wavefront kernel for the anti-diagonal / knight-move categories, the claimed-task
 * prev-row kernel, the inverted-L kernel; paper_conf_ipps_kumark15_b200/csrc/*.cuh) for the
 * user's functor inside the user's own translation unit.  The compiled-in f's of liblddp.so use
 * the same kernels (and faster specialised ones); nothing here runs on the CPU.
 *
 * The functor (all members static, device code):
 *
 *   struct MyF {
 *     using T  = int32_t;       // cell type: int32_t or float
 *     using In = int32_t;       // per-cell input type (32-bit), read by load()
 *     static constexpr uint32_t kMask = LDDP_NB_L | LDDP_NB_UL | LDDP_NB_U;   // contributing set
 *     static constexpr int kScore = lddp_user::SCORE_LAST_CELL;   // optional (default: none)
 *     __device__ static In load(const void* user, int64_t i, int64_t j);    // input of cell (i, j)
 *     __device__ static T top(const void* user, int64_t j);     // row -1 at column j, -1 <= j <= cols
 *     __device__ static T left(const void* user, int64_t i);    // column -1 at row i
 *     __device__ static T right(const void* user, int64_t i);   // column `cols` at row i (read via UR)
 *     __device__ static T f(T L, T UL, T U, T UR, In in, int64_t i, int64_t j);   // the cell
 *   };
 *
 * `user` is the device pointer given in Problem::user (the user's own input arrays); f receives
 * the four representative neighbours RS(i,j) [L90] whatever its mask (the ones outside kMask are
 * unspecified and must not influence the result).
 *
 * Validation (Table I): kMask must be a non-empty subset of RS (static_assert); the requested
 * category must order every dependency in kMask (lddp_category_covers of the library, same rule
 * as lddp_plan): otherwise LDDP_ERR_CATEGORY_MISMATCH.  Knight-move orders all 15 sets, so every
 * f has at least one category.  Categories: PREV_ROW, ANTI_DIAGONAL, KNIGHT_MOVE, INVERTED_L
 * (the twins VERTICAL / MINVERTED_L are reached through their general categories: knight-move).
 *
 * Outputs (device pointers, NULL = not requested): score (kScore: last cell, or minimum of the
 * last row), last_row (cols), last_col (rows; not for PREV_ROW), table (rows x table_pitch).
 * Workspace: workspace_bytes(problem) bytes of device memory, zeroed once before first use.
 * Errors are lddp_status codes; nothing throws.  Link with liblddp.so (host-side validation).
 */
#pragma once
#include <atomic>
#include <cstdint>
#include <cuda_runtime.h>

#include "lddp.h"
#include "../paper_conf_ipps_kumark15_b200/csrc/invl.cuh"
#include "../paper_conf_ipps_kumark15_b200/csrc/prevrow.cuh"
#include "../paper_conf_ipps_kumark15_b200/csrc/wavefront_launch.cuh"

namespace lddp_user {

enum { SCORE_NONE = lddp::SCORE_NONE, SCORE_LAST_CELL = lddp::SCORE_LAST_CELL, SCORE_ROW_MIN = lddp::SCORE_ROW_MIN };

struct Problem {
  int64_t rows = 0, cols = 0;
  int32_t category = LDDP_CAT_KNIGHT_MOVE;   // lddp_category
  int32_t device = 0;
  const void* user = nullptr;                // handed to load / top / left / right
  void* score = nullptr;
  void* last_row = nullptr;
  void* last_col = nullptr;
  void* table = nullptr;
  int64_t table_pitch = 0;                   // elements
};

namespace detail {

template <class UF, class = void>
struct ScoreOf { static constexpr int value = SCORE_NONE; };
template <class UF>
struct ScoreOf<UF, decltype(void(UF::kScore))> { static constexpr int value = UF::kScore; };

// The library's cell-functor interface (cellfn.cuh) around the user's functor: per-cell inputs
// arrive through the kGridIn path (load), FillParams::grid carries Problem::user.
template <class UF>
struct Cell {
  using T = typename UF::T;
  using RowCtx = int32_t;
  using ColCtx = int32_t;
  using GridT = typename UF::In;
  using OutT = T;
  static_assert(sizeof(T) == 4 && sizeof(GridT) == 4, "32-bit cells and inputs");
  static_assert(UF::kMask >= 1u && UF::kMask <= 15u, "kMask: a non-empty subset of {L, UL, U, UR} [L90]");
  static constexpr uint32_t kMask = UF::kMask;
  static constexpr bool kGridIn = true;
  static constexpr int kScore = ScoreOf<UF>::value;
  __device__ static RowCtx row_ctx(const lddp::FillParams&, int64_t) { return 0; }
  __device__ static ColCtx col_ctx(const lddp::FillParams&, int) { return 0; }
  __device__ static T top(const lddp::FillParams& p, int gc) { return UF::top(p.grid, gc); }
  __device__ static T left(const lddp::FillParams& p, int64_t i) { return UF::left(p.grid, i); }
  __device__ static T right(const lddp::FillParams& p, int64_t i) { return UF::right(p.grid, i); }
  __device__ static GridT load(const lddp::FillParams& p, int64_t i, int c) { return UF::load(p.grid, i, c); }
  __device__ static void prefetch_l1(const lddp::FillParams&, int64_t, int) {}
  __device__ __forceinline__ static T f(T L, T UL, T U, T UR, RowCtx, ColCtx, GridT in, int64_t i, int gc, int,
                                        OutT& o) {
    const T v = UF::f(L, UL, U, UR, in, i, (int64_t)gc);
    o = v;
    return v;
  }
};

inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }
inline uint64_t next_epoch() {
  static std::atomic<uint64_t> e{1u << 20};   // distinct from the library's own counter range
  return e.fetch_add(1) + 1;
}

// Geometry of the generic kernels (the same choices as liblddp.so's planner for them).
struct Geom {
  int kind;            // 0 wavefront (anti-diagonal / knight), 1 prev-row, 2 inverted-L
  int R, SIG, E;
  int64_t strip_rows, row0;
  int nstrips, nchunks, nblocks, nbands;
  int64_t bnd_stride;
  size_t off_prog, off_bnd, ws_bytes;
};

template <class UF>
inline Geom geometry(const Problem& pb) {
  Geom g{};
  const size_t cb = sizeof(typename UF::T);
  if (pb.category == LDDP_CAT_ANTI_DIAGONAL || pb.category == LDDP_CAT_KNIGHT_MOVE) {
    g.kind = 0;
    const bool knight = pb.category == LDDP_CAT_KNIGHT_MOVE;
    g.R = knight ? 1 : 4;
    g.SIG = knight ? 2 : 0;
    g.E = 2;
    g.strip_rows = (int64_t)lddp::kWfWarps * 32 * g.R;
    g.nstrips = (int)((pb.rows + g.strip_rows - 1) / g.strip_rows);
    g.row0 = pb.rows - (int64_t)g.nstrips * g.strip_rows;
    g.nchunks = (int)((pb.cols + 33 + 31) / 32);
    g.bnd_stride = (int64_t)g.nchunks * 32;
    g.off_prog = 64;
    g.off_bnd = align_up(g.off_prog + (size_t)(g.nstrips > 1 ? g.nstrips : 1) * 8, 256);
    g.ws_bytes = g.off_bnd + (size_t)(g.nstrips > 1 ? g.nstrips : 1) * g.bnd_stride * cb;
  } else if (pb.category == LDDP_CAT_PREV_ROW) {
    g.kind = 1;
    g.nblocks = (int)((pb.cols + 32 * lddp::kPrevV - 1) / (32 * lddp::kPrevV));
    g.nbands = (int)((pb.rows + lddp::kPrevBandRows - 1) / lddp::kPrevBandRows);
    g.bnd_stride = pb.cols > 1 ? pb.cols : 1;
    g.off_prog = 64;
    g.off_bnd = align_up(g.off_prog + (size_t)(g.nblocks > 1 ? g.nblocks : 1) * 16, 256);
    g.ws_bytes = g.off_bnd + (size_t)lddp::kPrevRing * g.bnd_stride * cb;
  } else {
    g.kind = 2;
    g.ws_bytes = 64;
  }
  return g;
}

}  // namespace detail

// Table I validation of a functor for a category (host; no GPU needed).
template <class UF>
inline lddp_status check(int32_t category) {
  if (category < LDDP_CAT_PREV_ROW || category > LDDP_CAT_INVERTED_L) return LDDP_ERR_UNSUPPORTED;
  int32_t covers = 0, pattern = -1;
  lddp_status st = lddp_classify(UF::kMask, &pattern);
  if (st != LDDP_OK) return st;
  st = lddp_category_covers(category, UF::kMask, &covers);
  if (st != LDDP_OK) return st;
  return covers ? LDDP_OK : LDDP_ERR_CATEGORY_MISMATCH;
}

template <class UF>
inline size_t workspace_bytes(const Problem& pb) {
  return detail::geometry<UF>(pb).ws_bytes;
}

// Enqueue one dependency-ordered fill of the user's f on `stream` (one persistent kernel).
template <class UF>
inline lddp_status fill(const Problem& pb, void* workspace, cudaStream_t stream) {
  using C = detail::Cell<UF>;
  lddp_status st = check<UF>(pb.category);
  if (st != LDDP_OK) return st;
  if (pb.rows < 0 || pb.cols < 0 || pb.cols > 0x7fff0000) return LDDP_ERR_SHAPE;
  if (pb.rows == 0 || pb.cols == 0) return LDDP_OK;
  if (workspace == nullptr) return LDDP_ERR_INVALID_ARG;
  if (pb.last_col != nullptr && pb.category == LDDP_CAT_PREV_ROW) return LDDP_ERR_UNSUPPORTED;
  if (pb.table != nullptr && pb.table_pitch < pb.cols) return LDDP_ERR_SHAPE;
  const detail::Geom g = detail::geometry<UF>(pb);
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, pb.device) != cudaSuccess) return LDDP_ERR_CUDA;
  lddp::FillParams p{};
  p.grid = pb.user;
  p.rows = pb.rows;
  p.cols = (int32_t)pb.cols;
  p.cols_total = (int32_t)pb.cols;
  p.is_last_rank = 1;
  p.score = pb.score;
  p.last_row = pb.last_row;
  p.last_col = pb.last_col;
  p.table = pb.table;
  p.table_pitch = pb.table_pitch;
  p.ctl = workspace;
  p.prog = reinterpret_cast<uint64_t*>(static_cast<char*>(workspace) + g.off_prog);
  p.bnd = static_cast<char*>(workspace) + g.off_bnd;
  p.bnd_stride = g.bnd_stride;
  p.epoch = detail::next_epoch();
  p.timeout_ns = 30ull * 1000000000ull;
  p.one = 1;
  p.spin_polls = 256;
  p.diag_lo = -(pb.rows - 1);   // inverted-L: every diagonal d = j - i
  p.diag_hi = pb.cols;
  cudaError_t e = cudaSuccess;
  const bool tab = pb.table != nullptr;
  // check() guarantees the category orders kMask, so only the kernels whose schedule can run
  // this f are instantiated (if constexpr) and reached
  if (g.kind == 0) {
    p.nstrips = g.nstrips;
    p.nchunks = g.nchunks;
    p.row0 = g.row0;
    p.strip_rows = g.strip_rows;
    const int grid = g.nstrips < 2 * sms ? g.nstrips : 2 * sms;
    if (pb.category == LDDP_CAT_KNIGHT_MOVE) {
      e = tab ? lddp::wf_launch<C, 1, 2, 2, lddp::kWfWarps, true, 1>(p, grid, stream)
              : lddp::wf_launch<C, 1, 2, 2, lddp::kWfWarps, false, 1>(p, grid, stream);
    } else {
      if constexpr (!(UF::kMask & LDDP_NB_UR))
        e = tab ? lddp::wf_launch<C, 4, 0, 2, lddp::kWfWarps, true, 4>(p, grid, stream)
                : lddp::wf_launch<C, 4, 0, 2, lddp::kWfWarps, false, 4>(p, grid, stream);
    }
  } else if (g.kind == 1) {
    if constexpr (!(UF::kMask & LDDP_NB_L)) {
      p.nstrips = g.nbands;
      p.nblocks = g.nblocks;
      p.block_cols = 32 * lddp::kPrevV;
      p.halo = lddp::kPrevBandRows;
      const int64_t tasks = (int64_t)g.nblocks * g.nbands;
      int64_t grid = (tasks + 7) / 8;
      if (grid > 4 * (int64_t)sms) grid = 4 * (int64_t)sms;
      if (tab)
        lddp::prevrow_kernel<C, true><<<(int)grid, lddp::kPrevWarps * 32, 0, stream>>>(p);
      else
        lddp::prevrow_kernel<C, false><<<(int)grid, lddp::kPrevWarps * 32, 0, stream>>>(p);
      e = cudaGetLastError();
    }
  } else {
    if constexpr (UF::kMask == LDDP_NB_UL) {
      const int64_t warps = (pb.rows + pb.cols - 1 + 31) / 32;
      int64_t grid = (warps + lddp::kInvlWarps - 1) / lddp::kInvlWarps;
      if (grid > 16 * (int64_t)sms) grid = 16 * (int64_t)sms;
      if (tab)
        lddp::invl_kernel<C, true, false><<<(int)grid, lddp::kInvlWarps * 32, 0, stream>>>(p);
      else
        lddp::invl_kernel<C, false, false><<<(int)grid, lddp::kInvlWarps * 32, 0, stream>>>(p);
      e = cudaGetLastError();
    }
  }
  return e == cudaSuccess ? LDDP_OK : LDDP_ERR_CUDA;
}

}  // namespace lddp_user
