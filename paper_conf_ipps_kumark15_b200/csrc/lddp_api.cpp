// lddp_api.cpp -- C ABI of liblddp.so (include/lddp.h): classification (Table I), planning,
// workspace layout, fills (single GPU, host-buffer, multi-GPU column strips) and status.
//
// The planner is the paper's "framework maps the function to a pattern" step [L113]: the
// contributing set of the compiled-in f is checked against the requested category's schedule
// (Fig. 2 [L117-L122]); the launch geometry replaces the paper's empirical t_switch / t_share
// tuning [L288-L294] (there is no CPU share on B200: the fill is GPU-only).
#include "../../include/lddp.h"

#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>

#include "params.h"
#include "sync.cuh"

namespace lddp {
int wf_dispatch_lcs(int, int, bool, const FillParams*, int, cudaStream_t);
int wf_dispatch_lev(int, int, bool, const FillParams*, int, cudaStream_t);
int wf_dispatch_dtw(int, int, bool, const FillParams*, int, cudaStream_t);
int wf_dispatch_fs(int, int, bool, const FillParams*, int, cudaStream_t);
int wf_dispatch_minpath3(int, int, bool, const FillParams*, int, cudaStream_t);
int wf_dispatch_min2plus(int, int, bool, const FillParams*, int, cudaStream_t);
int wf_dispatch_diagmaxplus(int, int, bool, const FillParams*, int, cudaStream_t);
}  // namespace lddp
#include "ad_table.inc"

using lddp::FillParams;

namespace {

thread_local std::string g_last_error;
std::atomic<uint64_t> g_epoch{1};

lddp_status fail(lddp_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return s;
}

lddp_status cuda_fail(cudaError_t e, const char* what) {
  return fail(LDDP_ERR_CUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

#define CUDA_TRY(expr)                                              \
  do {                                                              \
    cudaError_t _e = (expr);                                        \
    if (_e != cudaSuccess) return cuda_fail(_e, #expr);             \
  } while (0)

// --------------------------------------------------------------------- Table I / Fig. 2
// Table I [L124-L142]: pattern of every non-empty contributing set (bits L=1, UL=2, U=4, UR=8).
const int kTable1[16] = {
    -1,                     // {} (not a valid f)
    LDDP_PAT_VERTICAL,      // {L}              [L133]
    LDDP_PAT_INVERTED_L,    // {UL}             [L129]
    LDDP_PAT_VERTICAL,      // {L,UL}           [L137]
    LDDP_PAT_HORIZONTAL,    // {U}              [L127]
    LDDP_PAT_ANTI_DIAGONAL, // {L,U}            [L135]
    LDDP_PAT_HORIZONTAL,    // {UL,U}           [L131]
    LDDP_PAT_ANTI_DIAGONAL, // {L,UL,U}         [L139]
    LDDP_PAT_MINVERTED_L,   // {UR}             [L126]
    LDDP_PAT_KNIGHT_MOVE,   // {L,UR}           [L134]
    LDDP_PAT_HORIZONTAL,    // {UL,UR}          [L130]
    LDDP_PAT_KNIGHT_MOVE,   // {L,UL,UR}        [L138]
    LDDP_PAT_HORIZONTAL,    // {U,UR}           [L128]
    LDDP_PAT_KNIGHT_MOVE,   // {L,U,UR}         [L136]
    LDDP_PAT_HORIZONTAL,    // {UL,U,UR}        [L132]
    LDDP_PAT_KNIGHT_MOVE,   // {L,UL,U,UR}      [L140]
};

// Dependencies each category's schedule strictly orders (Fig. 2 [L117-L122], 0-based t):
//   prev-row t=i: UL, U, UR (t-1); anti-diagonal t=i+j: L (t-1), UL (t-2), U (t-1);
//   knight-move t=2i+j: L (t-1), UL (t-3), U (t-2), UR (t-1); inverted-L t=min(i,j): UL only.
uint32_t category_allows(int cat) {
  switch (cat) {
    case LDDP_CAT_PREV_ROW: return LDDP_NB_UL | LDDP_NB_U | LDDP_NB_UR;
    case LDDP_CAT_ANTI_DIAGONAL: return LDDP_NB_L | LDDP_NB_UL | LDDP_NB_U;
    case LDDP_CAT_KNIGHT_MOVE: return LDDP_NB_L | LDDP_NB_UL | LDDP_NB_U | LDDP_NB_UR;
    case LDDP_CAT_INVERTED_L: return LDDP_NB_UL;
    case LDDP_CAT_VERTICAL: return LDDP_NB_L | LDDP_NB_UL;     // t = j: L (t-1), UL (t-1)
    case LDDP_CAT_MINVERTED_L: return LDDP_NB_UR;              // t = min(i, W-1-j): UR only
    default: return 0;
  }
}

uint32_t func_mask(int f) {
  switch (f) {
    case LDDP_F_LCS: return LDDP_NB_L | LDDP_NB_UL | LDDP_NB_U;
    case LDDP_F_DTW: return LDDP_NB_L | LDDP_NB_UL | LDDP_NB_U;
    case LDDP_F_FS_DITHER: return LDDP_NB_L | LDDP_NB_UL | LDDP_NB_U | LDDP_NB_UR;
    case LDDP_F_MIN_PATH3: return LDDP_NB_UL | LDDP_NB_U | LDDP_NB_UR;
    case LDDP_F_DIAG_MAXPLUS: return LDDP_NB_UL;
    case LDDP_F_MIN2_PLUS: return LDDP_NB_UL | LDDP_NB_U;
    case LDDP_F_LEVENSHTEIN: return LDDP_NB_L | LDDP_NB_UL | LDDP_NB_U;
    case LDDP_F_MIN2_PLUS_V: return LDDP_NB_L | LDDP_NB_UL;
    case LDDP_F_ANTIDIAG_MAXPLUS: return LDDP_NB_UR;
    default: return 0;
  }
}

bool seq_func(int f) { return f == LDDP_F_LCS || f == LDDP_F_DTW || f == LDDP_F_LEVENSHTEIN; }
size_t cell_bytes(int) { return 4; }   // int32 or binary32 cells for every f
size_t seq_elt_bytes(int f) { return f == LDDP_F_DTW ? 4 : 1; }
size_t grid_elt_bytes(int f) { return f == LDDP_F_FS_DITHER ? 1 : 4; }
size_t table_elt_bytes(int f) { return f == LDDP_F_FS_DITHER ? 1 : 4; }

int wf_dispatch(int func, int op, int variant, bool table, const FillParams* p, int grid,
                cudaStream_t s) {
  switch (func) {
    case LDDP_F_LCS: return lddp::wf_dispatch_lcs(op, variant, table, p, grid, s);
    case LDDP_F_LEVENSHTEIN: return lddp::wf_dispatch_lev(op, variant, table, p, grid, s);
    case LDDP_F_DTW: return lddp::wf_dispatch_dtw(op, variant, table, p, grid, s);
    case LDDP_F_FS_DITHER: return lddp::wf_dispatch_fs(op, variant, table, p, grid, s);
    case LDDP_F_MIN_PATH3: return lddp::wf_dispatch_minpath3(op, variant, table, p, grid, s);
    case LDDP_F_MIN2_PLUS: return lddp::wf_dispatch_min2plus(op, variant, table, p, grid, s);
    case LDDP_F_DIAG_MAXPLUS: return lddp::wf_dispatch_diagmaxplus(op, variant, table, p, grid, s);
    default: return -1;
  }
}

// Compiled adiag geometries (tools/gen_adiag.py): f, rows per lane R, lane lag E, warps per CTA W.
struct AdGeom {
  int func, R, E, W, S, TB;   // TB: TABLE output (one-warp strips, staging tile)
  cudaError_t (*launch)(const FillParams&, int, cudaStream_t);
};
const AdGeom kAdGeoms[] = {
LDDP_AD_TABLE_ROWS
};

// prev-row multi-GPU: edge pairs per slot and side in the comm window (>= HB of prevrow_cb and
// HBO of prevrow_hx)
constexpr int kHaloSide = 96;

bool ad_has_table(int func) {
  for (const auto& g : kAdGeoms)
    if (g.func == func && g.TB) return true;
  return false;
}

// Lane-systolic anti-diagonal geometry model, constants from the B200
// microbenchmarks in tools/micro (ad_step2.cu, lat.cu).  One warp's step (R cells per lane)
// costs t = max(chain / E, issue) + ~12 cycles: the chain is R dependent cell latencies plus
// the rotate SHFL (~27) and SEL; issue is ~4.2 instructions per cell; W / 4 warps share an SM
// sub-partition.  A fill takes about  waves x n x t  (every lane sweeps every column)  plus the
// pipeline lag: each warp starts 32E + ~12 steps after the one above, each CTA ~40 more (L2).
struct AdModel { double ipc, lat; };
AdModel ad_model(int func) {
  switch (func) {
    case LDDP_F_DTW: return {6.0, 4.0};          // FADD, FMNMX3, FADD; refit with the 4-group unroll (C2: R4 E2 best)
    case LDDP_F_LEVENSHTEIN: return {4.6, 14.0}; // ISETP, VIMNMX3, IMAD, SEL; chain of three
    default: return {4.2, 4.5};                  // LCS: ISETP, IMAD, IMAD.MOV, VIMNMX3; chain VIMNMX3
  }
}
double ad_cost(int func, int R, int E, int W, int S, int64_t m, int64_t n, int sms) {
  const AdModel md = ad_model(func);
  const double share = W / 4.0;   // warps per SM sub-partition
  // split (S = 1): two independent chains of R/2 cells per step, one more step of lane lag
  const double chain = md.lat * (S ? R / 2 : R) + 31.0;
  const double t = std::max(chain / E, share * md.ipc * R * (S ? 0.8 : 1.0)) + 12.0;
  const int64_t warps = (m + 32 * R - 1) / (32 * R);
  const int64_t cap = (int64_t)W * sms;
  const int64_t waves = (warps + cap - 1) / cap;
  const double lag = (double)warps * (32.0 * (E + S) + 12.0) + (double)((warps + W - 1) / W) * 40.0;
  return ((double)waves * (double)n + lag) * t;
}

// variant geometry: rows per lane R, intra-lane skew SIG, extra lag E
struct VariantGeom { int id, R, SIG, E; };
const VariantGeom kVariants[] = {
    // compiled wavefront geometries (the rest of the round-1 sweep measured slower and is no
    // longer built): anti-diagonal R4 chained (default, TABLE), R2 / R8 skewed; knight-move
    {0, 4, 0, 2}, {2, 2, 1, 1}, {3, 8, 1, 1}, {10, 1, 2, 2}, {11, 2, 2, 2}, {13, 1, 2, 1},
};
const VariantGeom* variant_geom(int id) {
  for (const auto& v : kVariants)
    if (v.id == id) return &v;
  return nullptr;
}
constexpr int kWfWarps = 4;           // must match wavefront_launch.cuh
constexpr int kPrevBandRows = 64;     // must match prevrow.cu
constexpr int kPrevBW = 128;
constexpr int kPrevRing = 4;
constexpr int kPrevThreads = 256;
constexpr int kInvlThreads = 128;   // must match invl.cu (kInvlWarps x 32)

int env_int(const char* name, int dflt) {
  const char* v = getenv(name);
  return (v && *v) ? atoi(v) : dflt;
}

}  // namespace

// ------------------------------------------------------------------------------ plan object
struct lddp_plan_s {
  lddp_desc desc;
  int kind;          // 0 = wavefront (anti-diag / knight), 1 = prev-row, 2 = inverted-L
  int variant;       // wavefront variant id
  int R, SIG, E, W;
  cudaError_t (*ad_launch)(const FillParams&, int, cudaStream_t);   // adiag geometry (kind 3)
  int sms;
  int grid;
  int occupancy;
  // wavefront geometry
  int64_t strip_rows;
  int nstrips;
  int nchunks;
  int64_t row0;
  int64_t bnd_stride;
  // prev-row geometry
  int nblocks;
  int nbands;
  int cb_variant;    // column-block persistent kernel (prevrow_cb.cu): -1 = not usable
  int cb_bw;         // its own columns per warp (block width)
  int cb_nw;         // warps per CTA
  int cb_nblocks;    // column blocks (one warp each)
  int hx_variant;    // hierarchical-exchange kernel (prevrow_hx.cu, no TABLE): -1 = not usable
  int hx_cw;         // its own columns per CTA
  int hx_ctas;       // CTAs (one per SM at most)
  // Floyd-Steinberg lane-systolic kernel (fsk.cu): used when the widths / pitches allow
  bool fsk;
  // symmetric twins: mInverted-L = the inverted-L kernel on the mirrored grid; Vertical = a
  // transpose + the prev-row plan of the transposed problem (inner), workspace offsets below
  bool mirror;
  lddp_plan_s* inner;
  size_t off_tab, off_inner;
  int fsk_W, fsk_E, fsk_R, fsk_nstrips;
  int64_t fsk_bnd_stride;
  // workspace layout (bytes)
  size_t off_prog, off_bnd, ws_bytes;
  // own workspace + host-fill staging
  void* own_ws;
  std::mutex mu;
  void* stage[6];
  size_t stage_bytes[6];
};

// Multi-GPU receive window (lddp.h): [ack 2 x S u64][flag 2 x S u64][value 2 x (m + 1) x 4 B]
struct lddp_comm_s {
  lddp_plan_t plan;
  int nranks, rank, device;
  void* window;          // this rank's window (device memory of this rank)
  size_t win_bytes;
  size_t off_flag, off_val, off_halo;   // off_halo: prev-row edges [from left 8 x kHaloSide][from right ...]
  int64_t nstrips, rows;
  void* next;            // rank+1's window (IPC-opened or in-process), NULL on the last rank
  void* prev;            // rank-1's window, NULL on rank 0
  bool next_ipc, prev_ipc;
  uint64_t fills;        // fill epoch k of the next lddp_fill_multi (rank-consistent call order)
};

namespace {

// Wavefront geometry for `cols` local columns.
void wf_geometry(lddp_plan_s* pl, int64_t cols) {
  pl->strip_rows = (int64_t)kWfWarps * 32 * pl->R;
  const int64_t m = pl->desc.rows;
  pl->nstrips = (int)((m + pl->strip_rows - 1) / pl->strip_rows);
  pl->row0 = m - (int64_t)pl->nstrips * pl->strip_rows;
  pl->nchunks = (int)((cols + 33 + 31) / 32);
  pl->bnd_stride = (int64_t)pl->nchunks * 32;
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// Caller must hold pl->mu.
lddp_status ensure_own_ws_locked(lddp_plan_t pl, void** ws, cudaStream_t stream) {
  if (*ws != nullptr) return LDDP_OK;
  if (pl->own_ws == nullptr) {
    CUDA_TRY(cudaMalloc(&pl->own_ws, std::max<size_t>(pl->ws_bytes, 64)));
    CUDA_TRY(cudaMemsetAsync(pl->own_ws, 0, std::max<size_t>(pl->ws_bytes, 64), stream));
  }
  *ws = pl->own_ws;
  return LDDP_OK;
}

lddp_status ensure_own_ws(lddp_plan_t pl, void** ws, cudaStream_t stream) {
  if (*ws != nullptr) return LDDP_OK;
  std::lock_guard<std::mutex> lk(pl->mu);
  return ensure_own_ws_locked(pl, ws, stream);
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
    else prev = -1;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// Score of an empty problem (one or both sequences empty): the boundary value.
lddp_status write_empty_outputs(lddp_plan_t pl, const lddp_outputs* out, cudaStream_t s) {
  const lddp_desc& d = pl->desc;
  if (out->score != nullptr && (d.outputs & LDDP_OUT_SCORE)) {
    if (d.func == LDDP_F_LCS) {
      int32_t v = 0;
      CUDA_TRY(cudaMemcpyAsync(out->score, &v, 4, cudaMemcpyHostToDevice, s));
    } else if (d.func == LDDP_F_LEVENSHTEIN) {
      int32_t v = (int32_t)std::max(d.rows, d.cols);
      CUDA_TRY(cudaMemcpyAsync(out->score, &v, 4, cudaMemcpyHostToDevice, s));
    } else if (d.func == LDDP_F_DTW) {
      float v = (d.rows == 0 && d.cols == 0) ? 0.0f : __builtin_inff();
      CUDA_TRY(cudaMemcpyAsync(out->score, &v, 4, cudaMemcpyHostToDevice, s));
    }
    // memcpy from a stack variable: make it synchronous with respect to the host
    CUDA_TRY(cudaStreamSynchronize(s));
  }
  // LCS / Lev / DTW with rows > 0 and cols == 0: last_col of an empty region is empty; with
  // rows == 0 and cols > 0 the region's last row is empty.  Nothing else to write.
  return LDDP_OK;
}

lddp_status check_inputs(lddp_plan_t pl, const lddp_inputs* in, const lddp_outputs* out) {
  const lddp_desc& d = pl->desc;
  if (in == nullptr || out == nullptr) return fail(LDDP_ERR_INVALID_ARG, "inputs/outputs is NULL");
  if (seq_func(d.func)) {
    if ((d.rows > 0 && in->a == nullptr) || (d.cols > 0 && in->b == nullptr))
      return fail(LDDP_ERR_INVALID_ARG, "sequence input a/b is NULL");
  } else {
    if (in->grid == nullptr) return fail(LDDP_ERR_INVALID_ARG, "grid input is NULL");
    if (in->grid_pitch < d.cols) return fail(LDDP_ERR_SHAPE, "grid_pitch < cols");
  }
  if ((d.outputs & LDDP_OUT_SCORE) && out->score == nullptr)
    return fail(LDDP_ERR_INVALID_ARG, "SCORE requested but outputs.score is NULL");
  if ((d.outputs & LDDP_OUT_LAST_ROW) && out->last_row == nullptr)
    return fail(LDDP_ERR_INVALID_ARG, "LAST_ROW requested but outputs.last_row is NULL");
  if ((d.outputs & LDDP_OUT_LAST_COL) && out->last_col == nullptr)
    return fail(LDDP_ERR_INVALID_ARG, "LAST_COL requested but outputs.last_col is NULL");
  if (d.outputs & LDDP_OUT_TABLE) {
    if (out->table == nullptr) return fail(LDDP_ERR_INVALID_ARG, "TABLE requested but outputs.table is NULL");
    if (out->table_pitch < d.cols) return fail(LDDP_ERR_SHAPE, "table_pitch < cols");
  }
  return LDDP_OK;
}

void fill_common(lddp_plan_t pl, const lddp_inputs* in, const lddp_outputs* out, void* ws,
                 FillParams& p) {
  const lddp_desc& d = pl->desc;
  memset(&p, 0, sizeof p);
  p.a = in->a;
  p.b = in->b;
  p.grid = in->grid;
  p.grid_pitch = in->grid_pitch;
  p.rows = d.rows;
  p.cols = (int32_t)d.cols;
  p.col0 = 0;
  p.cols_total = (int32_t)d.cols;
  p.param_c = d.param_c;
  p.outputs = d.outputs;
  p.is_last_rank = 1;
  p.score = (d.outputs & LDDP_OUT_SCORE) ? out->score : nullptr;
  p.last_row = (d.outputs & LDDP_OUT_LAST_ROW) ? out->last_row : nullptr;
  p.last_col = (d.outputs & LDDP_OUT_LAST_COL) ? out->last_col : nullptr;
  p.table = (d.outputs & LDDP_OUT_TABLE) ? out->table : nullptr;
  p.table_pitch = out->table_pitch;
  p.ctl = ws;
  p.prog = reinterpret_cast<uint64_t*>(static_cast<char*>(ws) + pl->off_prog);
  p.bnd = static_cast<char*>(ws) + pl->off_bnd;
  p.bnd_stride = pl->bnd_stride;
  p.epoch = g_epoch.fetch_add(1) + 1;
  p.timeout_ns = (uint64_t)env_int("LDDP_TIMEOUT_MS", 30000) * 1000000ull;
  p.nstrips = pl->kind == 1 ? pl->nbands : pl->nstrips;
  p.nchunks = pl->nchunks;
  p.row0 = pl->row0;
  p.strip_rows = pl->strip_rows;
  p.block_cols = kPrevBW;
  p.halo = kPrevBandRows;
  p.nblocks = pl->nblocks;
  p.debug = env_int("LDDP_DEBUG", 0);
  p.spin_polls = env_int("LDDP_SPIN", 256);
  p.one = 1;
  p.diag_lo = -(d.rows - 1);
  p.diag_hi = d.cols;
  p.batch = std::max(d.batch, 1);
  // debug trace buffer: LDDP_TRACE=<device pointer as decimal>:<chunks per row>
  if (const char* tr = getenv("LDDP_TRACE")) {
    unsigned long long ptr = 0;
    int chunks = 0;
    if (sscanf(tr, "%llu:%d", &ptr, &chunks) == 2) {
      p.trace = reinterpret_cast<uint64_t*>(ptr);
      p.trace_chunks = chunks;
    }
  }
}

lddp_status launch(lddp_plan_t pl, const FillParams& p, cudaStream_t s) {
  cudaError_t e = cudaSuccess;
  if (pl->kind == 0 && pl->fsk && p.grid_pitch % 16 == 0 && p.table_pitch % 16 == 0 &&
      ((reinterpret_cast<uintptr_t>(p.grid) | reinterpret_cast<uintptr_t>(p.table)) & 15) == 0) {
    FillParams q = p;
    q.nstrips = pl->fsk_nstrips;
    q.bnd_stride = pl->fsk_bnd_stride;
    q.batch = std::max(q.batch, 1);
    const int fg = env_int("LDDP_FSK_GRID", 0);
    // one warp per SM for one image (measured best); up to one per SMSP for a batch
    const int gdef = pl->sms * std::min(q.batch, 4);
    e = lddp::launch_fsk(q, pl->fsk_W, pl->fsk_E, pl->fsk_R, std::min(fg > 0 ? fg : gdef, pl->fsk_nstrips * q.batch), s);
    if (e == cudaErrorInvalidValue)
      return fail(LDDP_ERR_UNSUPPORTED, "fsk W=%d E=%d R=%d not compiled", pl->fsk_W, pl->fsk_E, pl->fsk_R);
  } else if (pl->kind == 0 && pl->desc.batch > 1) {
    return fail(LDDP_ERR_UNSUPPORTED, "batched FS: grid / table rows must be 16-byte aligned with pitches %% 16 == 0");
  } else if (pl->kind == 0) {
    int grid = std::min(pl->grid, p.nstrips);
    int r = wf_dispatch(pl->desc.func, 0, pl->variant, p.table != nullptr, &p, grid, s);
    if (r < 0) return fail(LDDP_ERR_UNSUPPORTED, "wavefront variant %d not compiled for f=%d", pl->variant, pl->desc.func);
    e = (cudaError_t)r;
  } else if (pl->kind == 3) {
    int grid = std::min(pl->grid, p.nstrips);
    e = pl->ad_launch(p, grid, s);
  } else if (pl->kind == 4 && (reinterpret_cast<uintptr_t>(p.b) & 3) == 0) {
    int grid = std::min(pl->grid, p.nstrips);
    e = lddp::launch_lcs16(p, pl->R, pl->E, grid, s);
  } else if (pl->kind == 4) {
    // b not 4-byte aligned (lcs16 copies it in 4-byte granules): the 32-bit adiag kernel
    FillParams q = p;
    q.nstrips = (int)((pl->desc.rows + 191) / 192);
    q.row0 = pl->desc.rows - (int64_t)q.nstrips * 192;
    q.strip_rows = 192;
    q.bnd_stride = (int64_t)std::max((q.cols + 31) / 32, 1) * 32;
    e = lddp::ad_lcs_r6e2w1(q, std::min(q.nstrips, pl->sms * 8), s);
  } else if (pl->kind == 1 && pl->hx_variant >= 0 && p.grid_pitch % 4 == 0 && p.grid_pitch < ((int64_t)1 << 29) &&
             ((reinterpret_cast<uintptr_t>(p.grid) & 15) == 0) &&
             (p.table == nullptr || (p.table_pitch % 4 == 0 && p.table_pitch < ((int64_t)1 << 29) &&
                                     (reinterpret_cast<uintptr_t>(p.table) & 15) == 0))) {
    int dummy[3];
    e = lddp::launch_prevrow_hx(pl->desc.func, pl->hx_variant, p, false, dummy, s);
  } else if (pl->kind == 1 && pl->cb_variant >= 0 && (p.grid_pitch % 4 == 0) &&
             ((reinterpret_cast<uintptr_t>(p.grid) & 15) == 0)) {
    FillParams q = p;
    q.nblocks = pl->cb_nblocks;
    int dummy[2];
    e = lddp::launch_prevrow_cb(pl->desc.func, pl->cb_variant, q, pl->cb_nw, false, dummy, s);
  } else if (pl->kind == 1) {
    const int64_t ntasks = (int64_t)pl->nblocks * pl->nbands;
    FillParams q = p;
    // TMA streaming path: 32-bit costs, W % 4 == 0, 16-byte aligned rows (lddp.h documents the
    // fallback); block_cols = -1 selects it
    const bool tma = (q.cols % 4 == 0) && (q.grid_pitch % 4 == 0) &&
                     ((reinterpret_cast<uintptr_t>(q.grid) & 15) == 0) && env_int("LDDP_PREVROW_TMA", 1);
    int grid = (int)std::min<int64_t>(pl->grid, (ntasks + 7) / 8);
    if (tma) {
      // x2 CTAs of 4 warps; about two bands of tasks resident (more only spin on flags)
      q.block_cols = -1;
      const int64_t want = std::max<int64_t>(1, (2 * (int64_t)pl->nblocks + 7) / 8);
      grid = (int)std::max<int64_t>(1, std::min<int64_t>({(int64_t)pl->grid / 2, (ntasks + 7) / 8, want}));
      if (const char* g = getenv("LDDP_PREVROW_CTAS")) grid = std::max(1, atoi(g) / 2);
    }
    e = lddp::launch_prevrow(pl->desc.func, q, grid, s);
  } else if (pl->kind == 5) {
    // Vertical: grid (H x W) -> workspace (W x H), the transposed prev-row fill, table back
    lddp_plan_s* in = pl->inner;
    char* ws = static_cast<char*>(p.ctl);
    const int64_t H = pl->desc.rows, W = pl->desc.cols;
    int32_t* tg = reinterpret_cast<int32_t*>(ws + pl->off_bnd);
    e = lddp::launch_transpose_i32(static_cast<const int32_t*>(p.grid), p.grid_pitch, tg, H, H, W, s);
    if (e != cudaSuccess) return cuda_fail(e, "transpose launch");
    lddp_inputs din{};
    din.grid = tg;
    din.grid_pitch = H;
    lddp_outputs dout{};
    dout.score = p.score;
    dout.last_row = p.last_col;
    int32_t* tt = reinterpret_cast<int32_t*>(ws + pl->off_tab);
    if (p.table != nullptr) {
      dout.table = tt;
      dout.table_pitch = H;
    }
    FillParams q;
    fill_common(in, &din, &dout, ws + pl->off_inner, q);
    lddp_status st = launch(in, q, s);
    if (st != LDDP_OK) return st;
    if (p.table != nullptr) {
      e = lddp::launch_transpose_i32(tt, H, static_cast<int32_t*>(p.table), p.table_pitch, W, H, s);
      if (e != cudaSuccess) return cuda_fail(e, "transpose launch");
    }
    return LDDP_OK;
  } else {
    e = env_int("LDDP_INVL_TMA", 1) ? lddp::launch_invl_tma(p, pl->mirror, pl->sms, s) : cudaErrorNotSupported;
    if (e == cudaErrorNotSupported) e = lddp::launch_invl(pl->desc.func, p, pl->grid, pl->mirror, s);
  }
  if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
  return LDDP_OK;
}

}  // namespace

extern "C" {

int32_t lddp_abi_version(void) { return LDDP_ABI_VERSION; }

const char* lddp_status_string(lddp_status s) {
  switch (s) {
    case LDDP_OK: return "LDDP_OK";
    case LDDP_ERR_INVALID_ARG: return "LDDP_ERR_INVALID_ARG";
    case LDDP_ERR_SHAPE: return "LDDP_ERR_SHAPE";
    case LDDP_ERR_CATEGORY_MISMATCH: return "LDDP_ERR_CATEGORY_MISMATCH";
    case LDDP_ERR_UNSUPPORTED: return "LDDP_ERR_UNSUPPORTED";
    case LDDP_ERR_OUT_OF_MEMORY: return "LDDP_ERR_OUT_OF_MEMORY";
    case LDDP_ERR_CUDA: return "LDDP_ERR_CUDA";
    case LDDP_ERR_COMM: return "LDDP_ERR_COMM";
    case LDDP_ERR_TIMEOUT: return "LDDP_ERR_TIMEOUT";
    case LDDP_ERR_INTERNAL: return "LDDP_ERR_INTERNAL";
  }
  return "LDDP_ERR_UNKNOWN";
}

const char* lddp_last_error_message(void) { return g_last_error.c_str(); }

lddp_status lddp_func_mask(int32_t func, uint32_t* mask) {
  if (mask == nullptr) return fail(LDDP_ERR_INVALID_ARG, "mask is NULL");
  uint32_t m = func_mask(func);
  if (m == 0) return fail(LDDP_ERR_INVALID_ARG, "unknown func %d", func);
  *mask = m;
  return LDDP_OK;
}

lddp_status lddp_classify(uint32_t mask, int32_t* pattern) {
  if (pattern == nullptr) return fail(LDDP_ERR_INVALID_ARG, "pattern is NULL");
  if (mask == 0 || mask > 15) return fail(LDDP_ERR_INVALID_ARG, "contributing set must be a non-empty subset of RS(i,j)");
  *pattern = kTable1[mask];
  return LDDP_OK;
}

lddp_status lddp_category_covers(int32_t category, uint32_t mask, int32_t* covers) {
  if (covers == nullptr) return fail(LDDP_ERR_INVALID_ARG, "covers is NULL");
  if (category < 0 || category > 5) return fail(LDDP_ERR_INVALID_ARG, "unknown category %d", category);
  if (mask == 0 || mask > 15) return fail(LDDP_ERR_INVALID_ARG, "bad mask");
  *covers = (mask & ~category_allows(category)) == 0 ? 1 : 0;
  return LDDP_OK;
}

lddp_status lddp_plan(const lddp_desc* desc, lddp_plan_t* out) {
  try {
    if (desc == nullptr || out == nullptr) return fail(LDDP_ERR_INVALID_ARG, "desc/plan is NULL");
    *out = nullptr;
    const lddp_desc& d = *desc;
    const uint32_t fm = func_mask(d.func);
    if (fm == 0) return fail(LDDP_ERR_INVALID_ARG, "unknown func %d", d.func);
    if (d.category < 0 || d.category > 5) return fail(LDDP_ERR_INVALID_ARG, "unknown category %d", d.category);
    if (d.rows < 0 || d.cols < 0) return fail(LDDP_ERR_SHAPE, "negative shape");
    if (d.batch < 0) return fail(LDDP_ERR_INVALID_ARG, "negative batch");
    if (d.batch > 1 && d.func != LDDP_F_FS_DITHER)
      return fail(LDDP_ERR_UNSUPPORTED, "batch > 1 is supported for FS_DITHER (batched images) only");
    if (d.cols > (int64_t)0x7fff0000 || d.rows > ((int64_t)1 << 40)) return fail(LDDP_ERR_SHAPE, "shape too large");
    if (d.outputs & ~(LDDP_OUT_SCORE | LDDP_OUT_LAST_ROW | LDDP_OUT_LAST_COL | LDDP_OUT_TABLE))
      return fail(LDDP_ERR_INVALID_ARG, "unknown output bits 0x%x", d.outputs);
    if ((fm & ~category_allows(d.category)) != 0)
      return fail(LDDP_ERR_CATEGORY_MISMATCH,
                  "category %d does not order the contributing set 0x%x of f=%d (Table I)", d.category, fm, d.func);
    if (d.func == LDDP_F_FS_DITHER && !(d.outputs & LDDP_OUT_TABLE))
      return fail(LDDP_ERR_INVALID_ARG, "FS_DITHER writes the output image: request LDDP_OUT_TABLE");
    if ((d.outputs & LDDP_OUT_SCORE) &&
        (d.func == LDDP_F_FS_DITHER || d.func == LDDP_F_DIAG_MAXPLUS))
      return fail(LDDP_ERR_INVALID_ARG, "f=%d has no score output", d.func);
    if ((d.outputs & LDDP_OUT_LAST_COL) && d.category == LDDP_CAT_PREV_ROW)
      return fail(LDDP_ERR_UNSUPPORTED, "LAST_COL is not produced by the prev-row kernel");
    // the symmetric twins' f's run only in their own categories (on their twins' kernels)
    if ((d.func == LDDP_F_MIN2_PLUS_V) != (d.category == LDDP_CAT_VERTICAL) ||
        (d.func == LDDP_F_ANTIDIAG_MAXPLUS) != (d.category == LDDP_CAT_MINVERTED_L))
      return fail(LDDP_ERR_UNSUPPORTED, "f=%d in category %d: the twin f's MIN2_PLUS_V / ANTIDIAG_MAXPLUS run in "
                  "the VERTICAL / MINVERTED_L categories, and only those f's are compiled for them", d.func, d.category);
    if ((d.outputs & LDDP_OUT_LAST_ROW) && d.category == LDDP_CAT_VERTICAL)
      return fail(LDDP_ERR_UNSUPPORTED, "LAST_ROW is not produced by the vertical (transposed prev-row) path");
    if ((d.outputs & LDDP_OUT_SCORE) && d.func == LDDP_F_ANTIDIAG_MAXPLUS)
      return fail(LDDP_ERR_INVALID_ARG, "f=%d has no score output", d.func);
    if (d.func == LDDP_F_MIN_PATH3 && d.rows == 0 && d.cols > 0)
      return fail(LDDP_ERR_SHAPE, "MIN_PATH3 needs at least one row");

    lddp_plan_s* pl = new (std::nothrow) lddp_plan_s();
    if (pl == nullptr) return fail(LDDP_ERR_OUT_OF_MEMORY, "plan allocation");
    pl->desc = d;
    int dev = d.device;
    cudaDeviceProp prop;
    cudaError_t e = cudaGetDeviceProperties(&prop, dev);
    if (e != cudaSuccess) {
      delete pl;
      return cuda_fail(e, "cudaGetDeviceProperties");
    }
    pl->sms = prop.multiProcessorCount;
    DeviceGuard dg(dev);
    const bool table = (d.outputs & LDDP_OUT_TABLE) != 0;

    const char* kern_env = getenv("LDDP_KERNEL");
    const bool force_wf = kern_env != nullptr && strcmp(kern_env, "wavefront") == 0;
    const bool force_ad = kern_env != nullptr && strcmp(kern_env, "adiag") == 0;
    if (d.category == LDDP_CAT_ANTI_DIAGONAL && d.func == LDDP_F_LCS && !table && !force_wf && !force_ad) {
      // packed 16x2 LCS kernel (lcs16.cu): P row pairs per lane, lane lag E
      pl->kind = 4;
      // default P (measured on one B200): 6 (384-row strips) for C5-sized tables; 4 for tables of
      // <= 4096 rows, where pipeline fill / drain over few strips dominates (C1 0.065 -> 0.051 ms)
      pl->R = d.tile_rows > 0 ? (d.tile_rows + 1) / 2 : env_int("LDDP_L16_P", d.rows <= 4096 ? 4 : 6);
      pl->E = env_int("LDDP_L16_E", 2);
      pl->W = 1;
      pl->SIG = 0;
      if (!lddp::lcs16_compiled(pl->R, pl->E)) {   // nearest compiled P for this E (tile_rows hint)
        int best = -1;
        for (int P = 1; P <= 8; ++P)
          if (lddp::lcs16_compiled(P, pl->E) && (best < 0 || std::abs(P - pl->R) < std::abs(best - pl->R))) best = P;
        if (best > 0) pl->R = best;
      }
      if (!lddp::lcs16_compiled(pl->R, pl->E)) {
        const int P = pl->R, E = pl->E;
        delete pl;
        return fail(LDDP_ERR_UNSUPPORTED, "lcs16 P=%d E=%d not compiled", P, E);
      }
      pl->variant = -1;
      pl->occupancy = 1;
      pl->strip_rows = (int64_t)64 * pl->R;
      pl->nstrips = (int)((d.rows + pl->strip_rows - 1) / pl->strip_rows);
      pl->row0 = d.rows - (int64_t)pl->nstrips * pl->strip_rows;
      pl->nchunks = (int)((d.cols + 31) / 32);
      pl->bnd_stride = (int64_t)std::max(pl->nchunks, 1) * 32;
      int g = d.grid_ctas > 0 ? d.grid_ctas : env_int("LDDP_GRID_CTAS", 0);
      // grid = strip workers (warps), packed 4 per CTA: one warp per SM sub-partition
      pl->grid = g > 0 ? g : std::min(pl->nstrips, pl->sms * 4);
      pl->off_prog = 64;
      pl->off_bnd = 256;
      // boundary rows for lcs16's strips, or for the 192-row strips of the adiag fallback (b not
      // 4-byte aligned), whichever is more
      const int64_t fb_strips = (d.rows + 191) / 192;
      pl->ws_bytes = pl->off_bnd + (size_t)std::max<int64_t>(std::max(pl->nstrips, (int)fb_strips) - 1, 1) *
                                       pl->bnd_stride * 8;
    } else if (d.category == LDDP_CAT_ANTI_DIAGONAL && seq_func(d.func) && !force_wf &&
               (!table || ad_has_table(d.func))) {
      // lane-systolic anti-diagonal kernel (adiag.cuh)
      pl->kind = 3;
      int Rq = d.tile_rows > 0 ? d.tile_rows : env_int("LDDP_AD_R", 0);
      int Eq = env_int("LDDP_AD_E", 0);
      int Wq = d.tile_warps > 0 ? d.tile_warps : env_int("LDDP_AD_W", 0);
      int Sq = env_int("LDDP_AD_S", -1);
      // DTW: one warp per strip (every handoff through the global boundary rows, prefetched half
      // a chunk ahead) measured best on B200 (C2 0.93 -> 0.85 ms against 4-warp CTAs)
      if (Wq <= 0 && d.func == LDDP_F_DTW) Wq = 1;
      // Levenshtein (and LCS with LDDP_KERNEL=adiag): one-warp strips as well -- every handoff
      // through the global boundary rows, the next chunk's pairs prefetched inside the group loop
      // (measured best for C5 in round 1: 5.80 ms against 6.58 with 4-warp CTAs and shared rings);
      // with W = 1 forced, the cost model below only chooses among the W = 1 geometries
      if (Wq <= 0 && d.func != LDDP_F_DTW) {
        for (const auto& g : kAdGeoms)
          if (g.func == d.func && g.W == 1) { Wq = 1; break; }
      }
      double best = 1e300;
      pl->R = 0;
      for (const auto& g : kAdGeoms) {
        if (g.func != d.func) continue;
        if (Eq > 0 && g.E != Eq) continue;
        if (Wq > 0 && g.W != Wq) continue;
        if (Sq >= 0 && g.S != Sq) continue;
        if (Sq < 0 && g.S) continue;   // split geometries only on request: measured slower on B200 (C5 6.9 -> 11.6 ms)
        if (g.TB != (table ? 1 : 0)) continue;   // TABLE fills: the staging-tile instantiations
        double c = ad_cost(d.func, g.R, g.E, g.W, g.S, d.rows, std::max<int64_t>(d.cols, 1), pl->sms);
        if (Rq > 0) c += 1e200 * std::abs(g.R - Rq);   // nearest compiled R to the request
        if (getenv("LDDP_PLAN_DEBUG"))
          fprintf(stderr, "[lddp plan] f=%d R=%d E=%d W=%d S=%d cost=%.0f\n", (int)d.func, g.R, g.E, g.W, g.S, c);
        if (c < best) { best = c; pl->R = g.R; pl->E = g.E; pl->W = g.W; pl->SIG = g.S; pl->ad_launch = g.launch; }
      }
      if (pl->R == 0) {
        delete pl;
        return fail(LDDP_ERR_UNSUPPORTED, "no compiled adiag geometry for f=%d (E=%d W=%d)", d.func, Eq, Wq);
      }
      // pl->SIG carries the split flag (reported as "skew")
      pl->variant = -1;
      pl->occupancy = 1;
      pl->strip_rows = (int64_t)pl->W * 32 * pl->R;
      pl->nstrips = (int)((d.rows + pl->strip_rows - 1) / pl->strip_rows);
      pl->row0 = d.rows - (int64_t)pl->nstrips * pl->strip_rows;
      pl->nchunks = (int)((d.cols + 31) / 32);
      pl->bnd_stride = (int64_t)std::max(pl->nchunks, 1) * 32;   // (value, tag) pairs per strip row
      int g = d.grid_ctas > 0 ? d.grid_ctas : env_int("LDDP_GRID_CTAS", 0);
      // one-warp CTAs: enough of them for every strip to be resident at once
      pl->grid = g > 0 ? g : (pl->W == 1 ? std::min(pl->nstrips, pl->sms * 8) : pl->sms);
      pl->off_prog = 64;
      pl->off_bnd = 256;
      pl->ws_bytes = pl->off_bnd + (size_t)std::max(pl->nstrips - 1, 1) * pl->bnd_stride * 8;
    } else if (d.category == LDDP_CAT_ANTI_DIAGONAL || d.category == LDDP_CAT_KNIGHT_MOVE) {
      pl->kind = 0;
      const bool knight = d.category == LDDP_CAT_KNIGHT_MOVE;
      int rows = d.tile_rows > 0 ? d.tile_rows : env_int("LDDP_ROWS_PER_LANE", 0);
      int variant;
      if (knight) {
        int v_env = env_int("LDDP_WF_VARIANT", -1);
        variant = (rows == 2) ? 11 : 10;
        if (v_env == 10 || v_env == 11 || v_env == 13) variant = v_env;
      } else {
        int v_env = env_int("LDDP_WF_VARIANT", -1);
        if (v_env >= 0 && v_env != 10 && v_env != 11) variant = v_env;
        else if (rows == 2) variant = 2;
        else if (rows == 8) variant = 3;
        else variant = 0;
        // TABLE mode is compiled for variants 2 (R2, skewed: measured ~10 % faster for LCS /
        // Levenshtein / DTW 8192^2 TABLE fills, tools/table_time.py) and 0 (R4)
        if (table) {
          variant = (v_env == 0) ? 0 : 2;
          if (wf_dispatch(d.func, 2, variant, true, nullptr, 0, nullptr) < 0) variant = 0;   // R2 TABLE: seq f's only
        }
      }
      if (d.tile_warps != 0 && d.tile_warps != kWfWarps) {
        delete pl;
        return fail(LDDP_ERR_UNSUPPORTED, "tile_warps=%d (this build: %d)", d.tile_warps, kWfWarps);
      }
      const VariantGeom* vg = variant_geom(variant);
      if (vg == nullptr || wf_dispatch(d.func, 2, variant, table, nullptr, 0, nullptr) < 0) {
        delete pl;
        return fail(LDDP_ERR_UNSUPPORTED, "no compiled wavefront kernel for f=%d category=%d variant=%d table=%d",
                    d.func, d.category, variant, (int)table);
      }
      pl->variant = variant;
      pl->R = vg->R;
      pl->SIG = vg->SIG;
      pl->E = vg->E;
      pl->occupancy = wf_dispatch(d.func, 1, variant, table, nullptr, 0, nullptr);
      if (pl->occupancy <= 0) pl->occupancy = 1;
      wf_geometry(pl, d.cols);
      int g = d.grid_ctas > 0 ? d.grid_ctas : env_int("LDDP_GRID_CTAS", 0);
      pl->grid = g > 0 ? g : pl->sms * pl->occupancy;
      pl->off_prog = 64;
      pl->off_bnd = align_up(pl->off_prog + (size_t)std::max(pl->nstrips, 1) * 8, 256);
      pl->ws_bytes = pl->off_bnd + (size_t)std::max(pl->nstrips, 1) * pl->bnd_stride * cell_bytes(d.func);
      // FS: the lane-systolic knight kernel (fsk.cu) when the width is a multiple of 16 bytes
      // (16-byte image chunks); row pitches / alignment are checked per fill
      pl->fsk = false;
      if (knight && d.func == LDDP_F_FS_DITHER && table && d.cols > 0 && d.rows > 0 && d.cols % 16 == 0 &&
          env_int("LDDP_FSK", 1)) {
        pl->fsk = true;
        pl->fsk_W = env_int("LDDP_FSK_W", 1);   // measured best: one warp per strip (C3 1.87 -> 1.74 ms against 4)
        pl->fsk_E = env_int("LDDP_FSK_E", 1);
        pl->fsk_R = env_int("LDDP_FSK_R", 1);
        pl->fsk_nstrips = (int)((d.rows + 32 * pl->fsk_W * pl->fsk_R - 1) / (32 * pl->fsk_W * pl->fsk_R));
        pl->fsk_bnd_stride = ((d.cols + 31) / 32) * 32;   // (value, tag) pairs per boundary row
        pl->ws_bytes = std::max(pl->ws_bytes, pl->off_bnd + (size_t)pl->fsk_nstrips * pl->fsk_bnd_stride * 8 *
                                                  std::max(d.batch, 1));
      }
      if (d.batch > 1 && !pl->fsk) {
        delete pl;
        return fail(LDDP_ERR_UNSUPPORTED, "batched FS needs the fsk kernel (knight-move, cols %% 16 == 0, TABLE)");
      }
    } else if (d.category == LDDP_CAT_PREV_ROW) {
      pl->kind = 1;
      pl->nblocks = (int)((d.cols + kPrevBW - 1) / kPrevBW);
      pl->nbands = (int)((d.rows + kPrevBandRows - 1) / kPrevBandRows);
      pl->bnd_stride = std::max<int64_t>(d.cols, 1);
      pl->occupancy = 4;
      int g = d.grid_ctas > 0 ? d.grid_ctas : env_int("LDDP_GRID_CTAS", 0);
      pl->grid = g > 0 ? g : pl->sms * pl->occupancy;
      pl->off_prog = 64;
      pl->off_bnd = align_up(pl->off_prog + (size_t)std::max(pl->nblocks, 1) * 16, 256);
      pl->ws_bytes = pl->off_bnd + (size_t)kPrevRing * pl->bnd_stride * cell_bytes(d.func);
      // Column-block persistent kernel: every block co-resident (cooperative launch), W % 4 == 0
      // (16-byte cost segments; the row pitch / base alignment is checked per fill).
      pl->cb_variant = -1;
      // desc.band_rows = the trapezoid band height HB (rows between two halo exchanges): each
      // value maps to the compiled column-block geometry with that HB
      int cbv_def = 5;
      if (d.band_rows > 0) {
        const int hb[][2] = {{16, 13}, {32, 5}, {48, 17}, {64, 0}};
        cbv_def = -2;
        for (const auto& x : hb)
          if (x[0] == d.band_rows) cbv_def = x[1];
        if (cbv_def == -2) {
          delete pl;
          return fail(LDDP_ERR_UNSUPPORTED, "band_rows=%d: compiled prev-row band heights are 16, 32, 48, 64",
                      d.band_rows);
        }
      }
      const int cbv = env_int("LDDP_CB_VARIANT", cbv_def);
      const int cbnw = std::max(1, std::min(8, env_int("LDDP_CB_WARPS", 4)));
      if (cbv >= 0 && d.cols > 0 && d.rows > 0 && d.cols % 4 == 0) {
        int q[2] = {0, 0};
        FillParams dummy{};
        if (lddp::launch_prevrow_cb(d.func, cbv, dummy, cbnw, true, q, nullptr) == cudaSuccess && q[0] > 0) {
          const int64_t nbq = (d.cols + q[0] - 1) / q[0];
          const int64_t ctas = (nbq + cbnw - 1) / cbnw;
          if (q[1] > 0 && ctas <= (int64_t)q[1] * pl->sms) {
            pl->cb_variant = cbv;
            pl->cb_nw = cbnw;
            pl->cb_nblocks = (int)nbq;
            pl->cb_bw = q[0];
            // workspace: row minima (4 B per block) + edge pairs [nb][4][2][HB <= 64] x 8 B
            const size_t prog = align_up(64 + (size_t)nbq * 4, 256);
            pl->off_prog = 64;
            pl->off_bnd = std::max(pl->off_bnd, prog);
            pl->ws_bytes = std::max(pl->ws_bytes, pl->off_bnd + (size_t)nbq * 4 * 2 * 64 * 8);
          }
        } else {
          cudaGetLastError();
        }
      }
      // Hierarchical-exchange kernel for SCORE / LAST_ROW fills: CTAs of four
      // warps exchange inner halos through shared memory, outer halos through L2 every HBO rows.
      // desc.band_rows keeps selecting the prev-row_cb band height (it is that kernel's knob).
      pl->hx_variant = -1;
      // measured default (tools/gpu_hx5.sh, one B200): variant 2 (no lane ghosts, 64-row ring):
      // C4 2.00 -> 1.53 ms, C7 2.33 -> 1.55 ms
      const int hxv = env_int("LDDP_HX_VARIANT", 2);
      if (hxv >= 0 && d.band_rows <= 0 && d.cols > 0 && d.rows > 0 &&
          d.cols % 4 == 0 && d.rows < (int64_t)1 << 30) {
        int q[3] = {0, 0, 0};
        FillParams dummy{};
        if (lddp::launch_prevrow_hx(d.func, hxv, dummy, true, q, nullptr) == cudaSuccess && q[0] > 0) {
          const int64_t ctas = (d.cols + q[0] - 1) / q[0];
          if (q[1] > 0 && ctas <= (int64_t)q[1] * pl->sms) {
            pl->hx_variant = hxv;
            pl->hx_cw = q[0];
            pl->hx_ctas = (int)ctas;
            // workspace: per-CTA row minima + outer edge pairs [CTA][4 slots][2 sides][HBO] x 8 B,
            // or for one-way f's (no UR) [CTA][one slot per outer band][HBO]
            const size_t prog = align_up(64 + (size_t)ctas * 4, 256);
            const int64_t nob = (d.rows + q[2] - 1) / q[2];
            pl->off_prog = 64;
            pl->off_bnd = std::max(pl->off_bnd, prog);
            pl->ws_bytes = std::max(pl->ws_bytes, pl->off_bnd + (size_t)ctas * std::max<int64_t>(8, nob) * q[2] * 8);
          }
        } else {
          cudaGetLastError();
        }
      }
    } else if (d.category == LDDP_CAT_VERTICAL) {
      // Vertical = transpose of Horizontal [L111]: transpose the grid into the workspace, run the
      // prev-row plan of the transposed problem (its last row = our last column, its score =
      // ours), transpose a TABLE output back
      pl->kind = 5;
      lddp_desc t = d;
      t.rows = d.cols;
      t.cols = d.rows;
      t.category = LDDP_CAT_PREV_ROW;
      t.func = LDDP_F_MIN2_PLUS;
      t.outputs = (d.outputs & LDDP_OUT_SCORE) | ((d.outputs & LDDP_OUT_LAST_COL) ? LDDP_OUT_LAST_ROW : 0u) |
                  (d.outputs & LDDP_OUT_TABLE);
      lddp_status st = lddp_plan(&t, &pl->inner);
      if (st != LDDP_OK) {
        delete pl;
        return st;
      }
      const size_t cells = (size_t)std::max<int64_t>(d.rows, 0) * (size_t)std::max<int64_t>(d.cols, 0);
      pl->off_prog = 64;
      pl->off_bnd = 256;                                             // transposed grid (W x H)
      pl->off_tab = align_up(pl->off_bnd + cells * 4, 256);          // transposed table (TABLE)
      pl->off_inner = align_up(pl->off_tab + ((d.outputs & LDDP_OUT_TABLE) ? cells * 4 : 0), 256);
      pl->ws_bytes = pl->off_inner + std::max<size_t>(pl->inner->ws_bytes, 64);
      pl->grid = 1;
    } else {
      pl->kind = 2;
      pl->mirror = d.category == LDDP_CAT_MINVERTED_L;   // mInverted-L = mirror of Inverted-L [L111]
      const int64_t nd = d.rows + d.cols - 1;
      const int64_t warps = (nd + 31) / 32;
      const int64_t blocks = (warps + (kInvlThreads / 32) - 1) / (kInvlThreads / 32);
      pl->grid = (int)std::max<int64_t>(1, std::min<int64_t>(blocks, (int64_t)pl->sms * 16));   // every diagonal group resident
      pl->off_prog = 64;
      pl->off_bnd = 64;
      pl->ws_bytes = 64;
    }
    *out = pl;
    return LDDP_OK;
  } catch (...) {
    return fail(LDDP_ERR_INTERNAL, "exception in lddp_plan");
  }
}

lddp_status lddp_plan_destroy(lddp_plan_t pl) {
  if (pl == nullptr) return LDDP_OK;
  if (pl->inner) lddp_plan_destroy(pl->inner);
  DeviceGuard dg(pl->desc.device);
  if (pl->own_ws) cudaFree(pl->own_ws);
  for (int k = 0; k < 6; ++k)
    if (pl->stage[k]) cudaFree(pl->stage[k]);
  delete pl;
  return LDDP_OK;
}

lddp_status lddp_plan_workspace_size(lddp_plan_t pl, size_t* bytes) {
  if (pl == nullptr || bytes == nullptr) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
  *bytes = pl->ws_bytes;
  return LDDP_OK;
}

lddp_status lddp_plan_describe(lddp_plan_t pl, char* buf, size_t len) {
  if (pl == nullptr || buf == nullptr || len == 0) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
  static const char* kinds[] = {"wavefront", "prevrow", "invl", "adiag", "lcs16", "transpose+prevrow"};
  if (pl->kind == 5) {   // Vertical twin: describe the transposed prev-row plan it runs
    char inner[768];
    lddp_plan_describe(pl->inner, inner, sizeof inner);
    snprintf(buf, len, "{\"kernel\": \"transpose+prevrow\", \"workspace_bytes\": %zu, \"inner\": %s}", pl->ws_bytes, inner);
    return LDDP_OK;
  }
  const bool cb = pl->kind == 1 && pl->cb_variant >= 0;
  if (pl->kind == 1 && pl->hx_variant >= 0) {
    snprintf(buf, len,
             "{\"kernel\": \"prevrow_hx\", \"variant\": %d, \"warps\": 4, \"grid\": %d, \"sms\": %d, "
             "\"occupancy\": 1, \"cta_cols\": %d, \"workspace_bytes\": %zu, "
             "\"fallback\": \"prevrow_cb variant %d (TABLE, multi-GPU, unaligned grids)\"}",
             pl->hx_variant, pl->hx_ctas, pl->sms, pl->hx_cw, pl->ws_bytes, pl->cb_variant);
    return LDDP_OK;
  }
  if (pl->kind == 0 && pl->fsk) {
    snprintf(buf, len,
             "{\"kernel\": \"fsk\", \"variant\": -1, \"rows_per_lane\": %d, \"skew\": 2, \"extra_lag\": %d, "
             "\"warps\": %d, \"grid\": %d, \"sms\": %d, \"occupancy\": 1, \"strip_rows\": %d, "
             "\"strips\": %d, \"chunks\": %d, \"blocks\": 0, \"bands\": 0, \"workspace_bytes\": %zu, "
             "\"batch\": %d, \"fallback\": \"wavefront variant %d when pitches are not 16-byte multiples\"}",
             pl->fsk_R, pl->fsk_E, pl->fsk_W,
             std::min(pl->sms * std::min(std::max(pl->desc.batch, 1), 4), pl->fsk_nstrips * std::max(pl->desc.batch, 1)),
             pl->sms, 32 * pl->fsk_W * pl->fsk_R, pl->fsk_nstrips,
             (int)(pl->fsk_bnd_stride / 32), pl->ws_bytes, std::max(pl->desc.batch, 1), pl->variant);
    return LDDP_OK;
  }
  snprintf(buf, len,
           "{\"kernel\": \"%s\", \"variant\": %d, \"rows_per_lane\": %d, \"skew\": %d, \"extra_lag\": %d, "
           "\"warps\": %d, \"grid\": %d, \"sms\": %d, \"occupancy\": %d, \"strip_rows\": %lld, "
           "\"strips\": %d, \"chunks\": %d, \"blocks\": %d, \"bands\": %d, \"workspace_bytes\": %zu, "
           "\"mirror\": %d}",
           cb ? "prevrow_cb" : kinds[pl->kind], cb ? pl->cb_variant : pl->variant, pl->R, pl->SIG, pl->E,
           cb ? pl->cb_nw
              : (pl->kind == 0 ? kWfWarps + 2 : (pl->kind == 1 ? kPrevThreads / 32 : (pl->kind >= 3 ? pl->W : kInvlThreads / 32))),
           cb ? (pl->cb_nblocks + pl->cb_nw - 1) / pl->cb_nw : pl->grid,
           pl->sms, cb ? 1 : pl->occupancy, (long long)pl->strip_rows, pl->nstrips, pl->nchunks,
           cb ? pl->cb_nblocks : pl->nblocks, pl->nbands, pl->ws_bytes, pl->mirror ? 1 : 0);
  return LDDP_OK;
}

lddp_status lddp_workspace_init(lddp_plan_t pl, void* ws, void* stream) {
  if (pl == nullptr || ws == nullptr) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
  DeviceGuard dg(pl->desc.device);
  CUDA_TRY(cudaMemsetAsync(ws, 0, std::max<size_t>(pl->ws_bytes, 64), (cudaStream_t)stream));
  return LDDP_OK;
}

lddp_status lddp_fill(lddp_plan_t pl, const lddp_inputs* in, const lddp_outputs* out, void* ws,
                      void* stream) {
  try {
    if (pl == nullptr) return fail(LDDP_ERR_INVALID_ARG, "plan is NULL");
    lddp_status st = check_inputs(pl, in, out);
    if (st != LDDP_OK) return st;
    DeviceGuard dg(pl->desc.device);
    cudaStream_t s = (cudaStream_t)stream;
    const lddp_desc& d = pl->desc;
    if (d.rows == 0 || d.cols == 0) return write_empty_outputs(pl, out, s);
    if (d.func == LDDP_F_FS_DITHER) {
      // word-wide pixel access requirements (documented in lddp.h)
      if ((reinterpret_cast<uintptr_t>(in->grid) & 3) || (in->grid_pitch & 3) ||
          (reinterpret_cast<uintptr_t>(out->table) & 3) || (out->table_pitch & 3))
        return fail(LDDP_ERR_INVALID_ARG, "FS_DITHER needs 4-byte aligned image bases and pitches");
    }
    st = ensure_own_ws(pl, &ws, s);
    if (st != LDDP_OK) return st;
    FillParams p;
    fill_common(pl, in, out, ws, p);
    return launch(pl, p, s);
  } catch (...) {
    return fail(LDDP_ERR_INTERNAL, "exception in lddp_fill");
  }
}

lddp_status lddp_fill_host(lddp_plan_t pl, const lddp_inputs* hin, const lddp_outputs* hout,
                           void* stream) {
  try {
    if (pl == nullptr) return fail(LDDP_ERR_INVALID_ARG, "plan is NULL");
    lddp_status st = check_inputs(pl, hin, hout);
    if (st != LDDP_OK) return st;
    DeviceGuard dg(pl->desc.device);
    cudaStream_t s = (cudaStream_t)stream;
    const lddp_desc& d = pl->desc;
    std::lock_guard<std::mutex> lk(pl->mu);
    // device staging rows are re-pitched to 16-byte multiples whatever the host pitch (the FS /
    // prev-row fast paths need 16-byte aligned rows; the host pitch never reaches a kernel)
    const size_t gel = grid_elt_bytes(d.func), tel = table_elt_bytes(d.func);
    const size_t gdp = align_up((size_t)std::max<int64_t>(d.cols, 1) * gel, 16);
    const size_t tdp = align_up((size_t)std::max<int64_t>(d.cols, 1) * tel, 16);
    size_t need[6] = {0, 0, 0, 0, 0, 0};
    const int64_t Hb = d.rows * std::max(d.batch, 1);   // grid / table rows (batched FS images)
    if (seq_func(d.func)) {
      need[0] = d.rows * seq_elt_bytes(d.func);
      need[1] = d.cols * seq_elt_bytes(d.func);
    } else {
      need[2] = Hb * gdp;
    }
    need[3] = (d.outputs & LDDP_OUT_LAST_ROW) ? d.cols * cell_bytes(d.func) : 0;
    need[4] = (d.outputs & LDDP_OUT_LAST_COL) ? d.rows * cell_bytes(d.func) : 0;
    need[5] = (d.outputs & LDDP_OUT_TABLE) ? Hb * tdp + 16 : 16;
    for (int k = 0; k < 6; ++k) {
      if (need[k] > pl->stage_bytes[k]) {
        if (pl->stage[k]) cudaFree(pl->stage[k]);
        pl->stage[k] = nullptr;
        pl->stage_bytes[k] = 0;
        CUDA_TRY(cudaMalloc(&pl->stage[k], need[k]));
        pl->stage_bytes[k] = need[k];
      }
    }
    lddp_inputs din = *hin;
    lddp_outputs dout = *hout;
    if (need[0]) { CUDA_TRY(cudaMemcpyAsync(pl->stage[0], hin->a, need[0], cudaMemcpyHostToDevice, s)); din.a = pl->stage[0]; }
    if (need[1]) { CUDA_TRY(cudaMemcpyAsync(pl->stage[1], hin->b, need[1], cudaMemcpyHostToDevice, s)); din.b = pl->stage[1]; }
    if (need[2]) {
      CUDA_TRY(cudaMemcpy2DAsync(pl->stage[2], gdp, hin->grid, hin->grid_pitch * gel, d.cols * gel, Hb,
                                 cudaMemcpyHostToDevice, s));
      din.grid = pl->stage[2];
      din.grid_pitch = (int64_t)(gdp / gel);
    }
    if (d.outputs & LDDP_OUT_TABLE) dout.table_pitch = (int64_t)(tdp / tel);
    char* score_dev = static_cast<char*>(pl->stage[5]) + ((d.outputs & LDDP_OUT_TABLE) ? need[5] - 16 : 0);
    dout.score = hout->score ? score_dev : nullptr;
    dout.last_row = need[3] ? pl->stage[3] : nullptr;
    dout.last_col = need[4] ? pl->stage[4] : nullptr;
    dout.table = (d.outputs & LDDP_OUT_TABLE) ? pl->stage[5] : nullptr;
    void* ws = nullptr;
    st = ensure_own_ws_locked(pl, &ws, s);   // pl->mu is held
    if (st != LDDP_OK) return st;
    if (d.rows == 0 || d.cols == 0) {
      st = write_empty_outputs(pl, &dout, s);
    } else {
      FillParams p;
      fill_common(pl, &din, &dout, ws, p);
      st = launch(pl, p, s);
    }
    if (st != LDDP_OK) return st;
    if (hout->score && (d.outputs & LDDP_OUT_SCORE))
      CUDA_TRY(cudaMemcpyAsync(hout->score, score_dev, cell_bytes(d.func), cudaMemcpyDeviceToHost, s));
    if (need[3]) CUDA_TRY(cudaMemcpyAsync(hout->last_row, pl->stage[3], need[3], cudaMemcpyDeviceToHost, s));
    if (need[4]) CUDA_TRY(cudaMemcpyAsync(hout->last_col, pl->stage[4], need[4], cudaMemcpyDeviceToHost, s));
    if ((d.outputs & LDDP_OUT_TABLE) && d.rows > 0 && d.cols > 0)
      CUDA_TRY(cudaMemcpy2DAsync(hout->table, hout->table_pitch * tel, pl->stage[5], tdp, d.cols * tel, Hb,
                                 cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    return lddp_status_check(pl, ws, stream);
  } catch (...) {
    return fail(LDDP_ERR_INTERNAL, "exception in lddp_fill_host");
  }
}

lddp_status lddp_status_check(lddp_plan_t pl, void* ws, void* stream) {
  if (pl == nullptr) return fail(LDDP_ERR_INVALID_ARG, "plan is NULL");
  DeviceGuard dg(pl->desc.device);
  cudaStream_t s = (cudaStream_t)stream;
  CUDA_TRY(cudaStreamSynchronize(s));
  if (ws == nullptr) ws = pl->own_ws;
  if (ws == nullptr) return LDDP_OK;
  lddp::Control c;
  CUDA_TRY(cudaMemcpy(&c, ws, sizeof c, cudaMemcpyDeviceToHost));
  if (c.status != 0) {
    CUDA_TRY(cudaMemset(ws, 0, sizeof c));   // make the workspace usable again
    return fail((lddp_status)c.status, "device watchdog: a dependency wait exceeded LDDP_TIMEOUT_MS");
  }
  return LDDP_OK;
}

// ------------------------------------------------------------------------------ multi-GPU
lddp_status lddp_multi_partition(int64_t cols, int32_t nranks, int32_t rank, int64_t* c0, int64_t* c1) {
  if (c0 == nullptr || c1 == nullptr) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
  if (cols < 0 || nranks < 1 || rank < 0 || rank >= nranks) return fail(LDDP_ERR_INVALID_ARG, "bad partition request");
  *c0 = (int64_t)rank * cols / nranks;
  *c1 = (int64_t)(rank + 1) * cols / nranks;
  return LDDP_OK;
}

// The share of rank `rank` of `nranks` in a multi-GPU fill of this plan: columns [lo, hi) for
// column strips (anti-diagonal: near-equal; prev-row: whole column blocks of the column-block
// kernel), diagonals d = j - i in [lo, hi) for inverted-L diagonal shares (~1/P of the cells).
// lddp_fill_multi runs a prev-row plan on prevrow_hx when the plan has it and every rank gets at
// least one whole CTA strip (the partition is then CTA-aligned); prevrow_cb otherwise
static bool prev_multi_hx(const lddp_plan_s* pl, int nranks) {
  return pl->hx_variant >= 0 && (pl->desc.cols + pl->hx_cw - 1) / pl->hx_cw >= nranks;
}

static void plan_share(lddp_plan_t pl, int32_t nranks, int32_t rank, int64_t* lo, int64_t* hi) {
  const lddp_desc& d = pl->desc;
  const int64_t H = d.rows, W = d.cols;
  if (pl->kind == 2) {
    auto len = [&](int64_t dd) { return std::min(H, W - dd) - std::max<int64_t>(0, -dd); };
    const double total = (double)H * (double)W;
    const double lo_target = total * rank / nranks, hi_target = total * (rank + 1) / nranks;
    double acc = 0.0;
    int64_t dlo = -(H - 1), dhi = W;
    bool have_lo = rank == 0;
    for (int64_t dd = -(H - 1); dd < W; ++dd) {
      if (!have_lo && acc >= lo_target) { dlo = dd; have_lo = true; }
      acc += (double)len(dd);
      if (rank < nranks - 1 && acc >= hi_target) { dhi = dd + 1; break; }
    }
    if (!have_lo) dlo = W;
    if (H == 0 || W == 0) dlo = dhi = 0;
    *lo = dlo;
    *hi = std::max(dlo, dhi);
  } else if (pl->kind == 0 && pl->fsk) {
    const int64_t B = std::max(d.batch, 1);   // batched FS: images
    *lo = (int64_t)rank * B / nranks;
    *hi = (int64_t)(rank + 1) * B / nranks;
  } else if (pl->kind == 1 && (pl->cb_variant >= 0 || prev_multi_hx(pl, nranks))) {
    const int64_t BW = prev_multi_hx(pl, nranks) ? pl->hx_cw : pl->cb_bw;
    const int64_t NB = (W + BW - 1) / BW;
    const int64_t b0 = (int64_t)rank * NB / nranks, b1 = (int64_t)(rank + 1) * NB / nranks;
    *lo = std::min<int64_t>(b0 * BW, W);
    *hi = std::min<int64_t>(b1 * BW, W);
  } else {
    *lo = (int64_t)rank * W / nranks;
    *hi = (int64_t)(rank + 1) * W / nranks;
  }
}

lddp_status lddp_plan_partition(lddp_plan_t pl, int32_t nranks, int32_t rank, int64_t* lo, int64_t* hi) {
  if (pl == nullptr || lo == nullptr || hi == nullptr) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
  if (nranks < 1 || rank < 0 || rank >= nranks) return fail(LDDP_ERR_INVALID_ARG, "bad rank %d / %d", rank, nranks);
  plan_share(pl, nranks, rank, lo, hi);
  return LDDP_OK;
}

lddp_status lddp_comm_create(lddp_plan_t pl, int32_t nranks, int32_t rank, lddp_comm_t* out) {
  if (pl == nullptr || out == nullptr) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
  if (nranks < 1 || rank < 0 || rank >= nranks) return fail(LDDP_ERR_INVALID_ARG, "bad rank %d / %d", rank, nranks);
  const bool chains = pl->kind == 2 || (pl->kind == 0 && pl->fsk);   // inverted-L / batched FS: shares, no exchange
  const bool rows = pl->kind == 1;     // prev-row: column strips, two-way trapezoid halos
  if (rows && pl->cb_variant < 0)
    return fail(LDDP_ERR_UNSUPPORTED, "multi-GPU prev-row needs the column-block kernel (cols %% 4 == 0)");
  if (!chains && !rows && ((pl->kind != 3 && pl->kind != 4) || pl->desc.category != LDDP_CAT_ANTI_DIAGONAL))
    return fail(LDDP_ERR_UNSUPPORTED, "multi-GPU: anti-diagonal LCS / Levenshtein / DTW (column strips), prev-row "
                "(column strips, two-way halos), inverted-L / mInverted-L (diagonal shares) or FS (image shares)");
  if (!chains && pl->desc.cols < nranks) return fail(LDDP_ERR_SHAPE, "cols < nranks");
  DeviceGuard dg(pl->desc.device);
  lddp_comm_s* c = new (std::nothrow) lddp_comm_s();
  if (c == nullptr) return fail(LDDP_ERR_OUT_OF_MEMORY, "comm allocation");
  c->plan = pl;
  c->nranks = nranks;
  c->rank = rank;
  c->device = pl->desc.device;
  // strips of the widest geometry this plan can launch (lcs16 falls back to 192-row strips)
  c->nstrips = std::max<int64_t>(std::max<int64_t>(pl->nstrips, (pl->desc.rows + 191) / 192), 1);
  c->rows = pl->desc.rows;
  c->off_flag = align_up((size_t)2 * c->nstrips * 8, 256);
  c->off_val = c->off_flag + align_up((size_t)2 * c->nstrips * 8, 256);
  c->off_halo = align_up(c->off_val + (size_t)2 * (c->rows + 1) * 4, 256);
  c->win_bytes = c->off_halo + (size_t)2 * 8 * kHaloSide * 8;
  cudaError_t e = cudaMalloc(&c->window, c->win_bytes);
  if (e == cudaSuccess) e = cudaMemset(c->window, 0, c->win_bytes);
  if (e != cudaSuccess) {
    delete c;
    return cuda_fail(e, "window allocation");
  }
  c->fills = 0;
  *out = c;
  return LDDP_OK;
}

lddp_status lddp_comm_handle(lddp_comm_t c, uint8_t handle[LDDP_COMM_HANDLE_BYTES]) {
  if (c == nullptr || handle == nullptr) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
  static_assert(sizeof(cudaIpcMemHandle_t) <= LDDP_COMM_HANDLE_BYTES, "IPC handle size");
  DeviceGuard dg(c->device);
  cudaIpcMemHandle_t h;
  cudaError_t e = cudaIpcGetMemHandle(&h, c->window);
  if (e != cudaSuccess) return fail(LDDP_ERR_COMM, "cudaIpcGetMemHandle: %s", cudaGetErrorString(e));
  memset(handle, 0, LDDP_COMM_HANDLE_BYTES);
  memcpy(handle, &h, sizeof h);
  return LDDP_OK;
}

namespace {
lddp_status open_ipc(const uint8_t* handle, void** out) {
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof h);
  void* p = nullptr;
  cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) return fail(LDDP_ERR_COMM, "cudaIpcOpenMemHandle: %s", cudaGetErrorString(e));
  *out = p;
  return LDDP_OK;
}
lddp_status enable_peer(int dev, int peer) {
  if (peer == dev) return LDDP_OK;
  DeviceGuard dg(dev);
  int ok = 0;
  cudaDeviceCanAccessPeer(&ok, dev, peer);
  if (!ok) return fail(LDDP_ERR_COMM, "device %d cannot access peer %d", dev, peer);
  cudaError_t e = cudaDeviceEnablePeerAccess(peer, 0);
  if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
    return fail(LDDP_ERR_COMM, "cudaDeviceEnablePeerAccess: %s", cudaGetErrorString(e));
  cudaGetLastError();
  return LDDP_OK;
}
}  // namespace

lddp_status lddp_comm_connect(lddp_comm_t c, const uint8_t* next_handle, const uint8_t* prev_handle) {
  if (c == nullptr) return fail(LDDP_ERR_INVALID_ARG, "comm is NULL");
  if ((c->rank < c->nranks - 1) != (next_handle != nullptr))
    return fail(LDDP_ERR_INVALID_ARG, "rank %d of %d: next handle must be given iff a next rank exists", c->rank, c->nranks);
  if ((c->rank > 0) != (prev_handle != nullptr))
    return fail(LDDP_ERR_INVALID_ARG, "rank %d: previous handle must be given iff a previous rank exists", c->rank);
  DeviceGuard dg(c->device);
  if (next_handle != nullptr) {
    lddp_status st = open_ipc(next_handle, &c->next);
    if (st != LDDP_OK) return st;
    c->next_ipc = true;
  }
  if (prev_handle != nullptr) {
    lddp_status st = open_ipc(prev_handle, &c->prev);
    if (st != LDDP_OK) return st;
    c->prev_ipc = true;
  }
  return LDDP_OK;
}

lddp_status lddp_comm_connect_local(lddp_comm_t c, lddp_comm_t next, lddp_comm_t prev) {
  if (c == nullptr) return fail(LDDP_ERR_INVALID_ARG, "comm is NULL");
  if ((c->rank < c->nranks - 1) != (next != nullptr) || (c->rank > 0) != (prev != nullptr))
    return fail(LDDP_ERR_INVALID_ARG, "rank %d of %d: neighbours must be given iff they exist", c->rank, c->nranks);
  if (next != nullptr) {
    lddp_status st = enable_peer(c->device, next->device);
    if (st != LDDP_OK) return st;
    c->next = next->window;
    c->next_ipc = false;
  }
  if (prev != nullptr) {
    lddp_status st = enable_peer(c->device, prev->device);
    if (st != LDDP_OK) return st;
    c->prev = prev->window;
    c->prev_ipc = false;
  }
  return LDDP_OK;
}

lddp_status lddp_comm_destroy(lddp_comm_t c) {
  if (c == nullptr) return LDDP_OK;
  DeviceGuard dg(c->device);
  if (c->next_ipc && c->next) cudaIpcCloseMemHandle(c->next);
  if (c->prev_ipc && c->prev) cudaIpcCloseMemHandle(c->prev);
  if (c->window) cudaFree(c->window);
  delete c;
  return LDDP_OK;
}

lddp_status lddp_traceback(lddp_plan_t pl, const lddp_inputs* in, const void* table, int64_t table_pitch,
                           int32_t* path_i, int32_t* path_j, int64_t* path_len, void* stream) {
  try {
    if (pl == nullptr || in == nullptr || table == nullptr || path_i == nullptr || path_j == nullptr ||
        path_len == nullptr)
      return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
    const lddp_desc& d = pl->desc;
    if (d.func != LDDP_F_LCS && d.func != LDDP_F_LEVENSHTEIN && d.func != LDDP_F_DTW)
      return fail(LDDP_ERR_UNSUPPORTED, "traceback: LCS, Levenshtein or DTW only (f=%d)", d.func);
    if (table_pitch < d.cols) return fail(LDDP_ERR_INVALID_ARG, "table_pitch %lld < cols", (long long)table_pitch);
    if ((d.rows > 0 && in->a == nullptr) || (d.cols > 0 && in->b == nullptr))
      return fail(LDDP_ERR_INVALID_ARG, "traceback needs the fill's inputs a and b");
    DeviceGuard dg(d.device);
    cudaError_t e = lddp::launch_traceback(d.func, in->a, in->b, table, table_pitch, d.rows, d.cols, path_i, path_j,
                                           path_len, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "traceback launch");
    return LDDP_OK;
  } catch (...) {
    return fail(LDDP_ERR_INTERNAL, "exception in lddp_traceback");
  }
}

lddp_status lddp_fill_multi(lddp_plan_t pl, const lddp_inputs* in, const lddp_outputs* out,
                            void* ws, lddp_comm_t c, void* stream) {
  try {
    if (pl == nullptr || c == nullptr) return fail(LDDP_ERR_INVALID_ARG, "NULL argument");
    if (c->plan != pl) return fail(LDDP_ERR_INVALID_ARG, "comm was created for another plan");
    lddp_status st = check_inputs(pl, in, out);
    if (st != LDDP_OK) return st;
    const bool shares = pl->kind == 2 || (pl->kind == 0 && pl->fsk);   // no exchange between ranks
    if (!shares && c->rank < c->nranks - 1 && c->next == nullptr)
      return fail(LDDP_ERR_COMM, "rank %d is not connected to rank %d", c->rank, c->rank + 1);
    if (!shares && c->rank > 0 && c->prev == nullptr)
      return fail(LDDP_ERR_COMM, "rank %d is not connected to rank %d", c->rank, c->rank - 1);
    DeviceGuard dg(pl->desc.device);
    cudaStream_t s = (cudaStream_t)stream;
    const lddp_desc& d = pl->desc;
    if (pl->kind == 0 && pl->fsk) {
      // Batched FS (image-parallel): rank g fills images [g B / P, (g+1) B / P) of the batch
      // with one launch; images are independent, so nothing crosses ranks (weak scaling).
      int64_t b0 = 0, b1 = 0;
      plan_share(pl, c->nranks, c->rank, &b0, &b1);
      c->fills += 1;
      if (b1 <= b0 || d.rows == 0 || d.cols == 0) return LDDP_OK;
      st = ensure_own_ws(pl, &ws, s);
      if (st != LDDP_OK) return st;
      FillParams p;
      fill_common(pl, in, out, ws, p);
      p.grid = static_cast<const uint8_t*>(in->grid) + b0 * d.rows * in->grid_pitch;
      p.table = static_cast<uint8_t*>(out->table) + b0 * d.rows * out->table_pitch;
      p.batch = (int32_t)(b1 - b0);
      return launch(pl, p, s);
    }
    if (pl->kind == 2) {
      // Inverted-L (and its mirror twin): every diagonal chain is independent ([L203]); rank g
      // fills a contiguous share of the diagonals holding ~1/P of the cells, writing its chains'
      // ends into last_row / last_col and its cells into a TABLE output.  No communication.
      if (d.rows == 0 || d.cols == 0) return LDDP_OK;
      st = ensure_own_ws(pl, &ws, s);
      if (st != LDDP_OK) return st;
      FillParams p;
      fill_common(pl, in, out, ws, p);
      int64_t dlo = 0, dhi = 0;
      plan_share(pl, c->nranks, c->rank, &dlo, &dhi);
      p.diag_lo = dlo;
      p.diag_hi = dhi;
      c->fills += 1;
      if (p.diag_hi == p.diag_lo) return LDDP_OK;
      const int64_t warps = (p.diag_hi - p.diag_lo + 31) / 32;
      const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((warps + kInvlThreads / 32 - 1) / (kInvlThreads / 32),
                                                                   (int64_t)pl->sms * 16));
      cudaError_t e = env_int("LDDP_INVL_TMA", 1) ? lddp::launch_invl_tma(p, pl->mirror, pl->sms, s) : cudaErrorNotSupported;
      if (e == cudaErrorNotSupported) e = lddp::launch_invl(d.func, p, grid, pl->mirror, s);
      if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
      return LDDP_OK;
    }
    if (pl->kind == 1) {
      // Previous-row category: rank g owns a block-aligned column strip; the column-block kernel
      // exchanges its outer edges with the neighbour ranks every band (two-way trapezoid halos,
      // Table II case 2 [L265-L274]).  The grid is passed whole (the halos read HB columns of
      // the neighbours' costs); score = the minimum of this rank's last-row columns.
      if (d.rows == 0 || d.cols == 0) return LDDP_OK;
      if ((reinterpret_cast<uintptr_t>(in->grid) & 15) || (in->grid_pitch % 4))
        return fail(LDDP_ERR_UNSUPPORTED, "multi-GPU prev-row: 16-byte aligned grid, pitch %% 4 == 0");
      st = ensure_own_ws(pl, &ws, s);
      if (st != LDDP_OK) return st;
      int64_t c0 = 0, c1 = 0;
      plan_share(pl, c->nranks, c->rank, &c0, &c1);
      c->fills += 1;
      if (c1 <= c0) return LDDP_OK;
      FillParams p;
      fill_common(pl, in, out, ws, p);
      const size_t gel = grid_elt_bytes(d.func), tel = table_elt_bytes(d.func);
      p.grid = static_cast<const char*>(in->grid) + c0 * gel;
      p.cols = (int32_t)(c1 - c0);
      p.col0 = (int32_t)c0;
      p.cols_total = (int32_t)d.cols;
      if (p.last_row) p.last_row = static_cast<char*>(p.last_row) + c0 * cell_bytes(d.func);
      if (p.table) p.table = static_cast<char*>(p.table) + c0 * tel;
      p.nblocks = (int)((c1 - c0 + pl->cb_bw - 1) / pl->cb_bw);
      p.wepoch = c->fills;
      uint64_t* own = reinterpret_cast<uint64_t*>(static_cast<char*>(c->window) + c->off_halo);
      if (c->rank > 0) {
        p.halo_in_l = own;                                                                   // from left
        p.halo_out_l = reinterpret_cast<uint64_t*>(static_cast<char*>(c->prev) + c->off_halo) + 8 * kHaloSide;   // its "from right"
      }
      if (c->rank < c->nranks - 1) {
        p.halo_in_r = own + 8 * kHaloSide;                                                   // from right
        p.halo_out_r = reinterpret_cast<uint64_t*>(static_cast<char*>(c->next) + c->off_halo);            // its "from left"
      }
      cudaError_t e;
      if (prev_multi_hx(pl, c->nranks)) {
        // hierarchical-exchange kernel: CTA-aligned strips, the strip's outer CTA edges through
        // the windows every HBO rows (TABLE: 16-byte row stores)
        if (p.table != nullptr && ((p.table_pitch % 4) || (reinterpret_cast<uintptr_t>(p.table) & 15)))
          return fail(LDDP_ERR_UNSUPPORTED, "multi-GPU prev-row TABLE: 16-byte aligned table, pitch %% 4 == 0");
        int dummy3[3];
        e = lddp::launch_prevrow_hx(d.func, pl->hx_variant, p, false, dummy3, s);
      } else {
        int dummy2[2];
        e = lddp::launch_prevrow_cb(d.func, pl->cb_variant, p, pl->cb_nw, false, dummy2, s);
      }
      if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
      return LDDP_OK;
    }
    if (pl->desc.outputs & LDDP_OUT_TABLE) return fail(LDDP_ERR_UNSUPPORTED, "TABLE output is not supported by lddp_fill_multi");
    if (d.rows == 0) return LDDP_OK;
    st = ensure_own_ws(pl, &ws, s);
    if (st != LDDP_OK) return st;
    const int64_t n = d.cols;
    int64_t c0 = 0, c1 = 0;
    lddp_multi_partition(n, c->nranks, c->rank, &c0, &c1);
    FillParams p;
    fill_common(pl, in, out, ws, p);
    p.cols = (int32_t)(c1 - c0);
    p.col0 = (int32_t)c0;
    p.cols_total = (int32_t)n;
    p.nchunks = (int)((p.cols + 31) / 32);
    p.bnd_stride = (int64_t)std::max(p.nchunks, 1) * 32;
    const bool last = c->rank == c->nranks - 1;
    p.is_last_rank = last ? 1 : 0;
    if (p.last_row) p.last_row = static_cast<char*>(p.last_row) + c0 * cell_bytes(d.func);
    if (!last) {
      p.score = nullptr;
      p.last_col = nullptr;
    }
    // fill epoch k (1, 2, ...) and its window slot k & 1
    c->fills += 1;
    p.wepoch = c->fills;
    const int slot = (int)(p.wepoch & 1);
    const size_t val_slot = (size_t)slot * (c->rows + 1) * 4 + 4;   // element 0 = row -1
    auto win = [&](void* base, size_t off) { return reinterpret_cast<char*>(base) + off; };
    if (c->rank > 0) {
      p.lflag_in = reinterpret_cast<const uint64_t*>(win(c->window, c->off_flag)) + slot * c->nstrips;
      p.lcol_in = win(c->window, c->off_val + val_slot);
      p.ack_out = reinterpret_cast<uint64_t*>(win(c->prev, 0)) + slot * c->nstrips;
    }
    if (!last) {
      p.ack_in = reinterpret_cast<const uint64_t*>(win(c->window, 0)) + slot * c->nstrips;
      p.rflag_out = reinterpret_cast<uint64_t*>(win(c->next, c->off_flag)) + slot * c->nstrips;
      p.rcol_out = win(c->next, c->off_val + val_slot);
    }
    return launch(pl, p, s);
  } catch (...) {
    return fail(LDDP_ERR_INTERNAL, "exception in lddp_fill_multi");
  }
}

}  // extern "C"
