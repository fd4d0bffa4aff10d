// params.h -- kernel parameter block and launch entry points shared by the C-ABI layer
// (lddp_api.cpp, host C++) and the CUDA translation units.  Internal to liblddp.so.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace lddp {

struct FillParams {
  // problem (local to this rank for multi-GPU)
  const void* a;            // LCS/Lev: uint8[rows], DTW: float[rows]
  const void* b;            // LCS/Lev: uint8[cols_total], DTW: float[cols_total] (global)
  const void* grid;         // FS uint8 / int32 grid, rows x cols
  int64_t grid_pitch;       // elements
  int64_t rows;             // m / H
  int32_t cols;             // local number of f-evaluated columns
  int32_t col0;             // global column of local column 0 (multi-GPU), else 0
  int32_t cols_total;       // global number of columns
  int32_t param_c;
  uint32_t outputs;         // LDDP_OUT_* bits
  int32_t is_last_rank;     // 1 on single GPU / last rank (owns score + last_col)
  // outputs (device pointers, NULL if not requested)
  void* score;
  void* last_row;           // already offset by col0 on multi-GPU
  void* last_col;
  void* table;
  int64_t table_pitch;
  // workspace
  void* ctl;                // lddp::Control*
  uint64_t* prog;           // per strip / band progress flags (epoch << 32 | count)
  void* bnd;                // boundary rows between strips / bands
  int64_t bnd_stride;       // elements per strip row in bnd
  uint64_t epoch;           // workspace epoch (progress flags)
  uint64_t wepoch;          // multi-GPU window epoch (rank-consistent)
  uint64_t timeout_ns;
  // geometry
  int32_t nstrips;          // strips (anti-diag / knight) or bands (prev-row)
  int32_t nchunks;          // link chunks per strip (anti-diag / knight)
  int64_t row0;             // global row of strip 0's first row (<= 0: bottom-aligned strips)
  int64_t strip_rows;       // rows per strip / band
  // prev-row category
  int32_t block_cols;       // columns owned per CTA
  int32_t halo;             // trapezoid halo (= band rows)
  int32_t nblocks;          // column blocks
  // multi-GPU window (left boundary in, right column out), this fill's slot (lddp.h)
  const void* lcol_in;      // my window: rank g-1's right column, element i = row i (i >= -1)
  const uint64_t* lflag_in; // my window flags, one per strip
  uint64_t* ack_out;        // rank g-1's window acks (peer pointer): strip s read by me
  const uint64_t* ack_in;   // my window acks (written by rank g+1)
  void* rcol_out;           // rank g+1's window values (peer pointer), element i = row i, or NULL
  uint64_t* rflag_out;      // rank g+1's window flags (peer pointer) or NULL
  // debug trace (env LDDP_TRACE): globaltimer stamps per (strip, warp, chunk), or NULL
  uint64_t* trace;
  int32_t trace_chunks;     // chunks per (strip, warp) row of the trace
  int32_t one;              // always 1 (a run-time constant the compiler cannot fold)
  int32_t spin_polls;       // polls before a waiting warp starts to back off (env LDDP_SPIN)
  int32_t debug;            // env LDDP_DEBUG bits (development): 1 = adiag warps without handoffs
  int32_t workers;          // lcs16: persistent strip workers (warps); extra warps of the last CTA idle
  int32_t batch;            // fsk: independent images stacked along the rows (>= 1); claims are (strip, image) pairs
  int64_t diag_lo, diag_hi; // inverted-L: this rank's diagonals d = j - i in [diag_lo, diag_hi)
  // prev-row multi-GPU (column strips with two-way trapezoid halos, Table II case 2): edge pairs
  // [8 slots: fill parity x band mod 4][HB] exchanged with the neighbour ranks through the comm windows
  const uint64_t* halo_in_l;  // my window: rank g-1's right edge (read by my block 0)
  const uint64_t* halo_in_r;  // my window: rank g+1's left edge (read by my last block)
  uint64_t* halo_out_l;       // rank g-1's window: my left edge (peer pointer)
  uint64_t* halo_out_r;       // rank g+1's window: my right edge (peer pointer)
};

// Launch entry points (one per category family).  Return cudaError_t of the launch.
cudaError_t launch_wavefront(int func, int category, const FillParams& p, int rows_per_lane,
                             int warps, int grid, cudaStream_t stream);
cudaError_t launch_prevrow(int func, const FillParams& p, int grid, cudaStream_t stream);
// Column-block persistent prev-row kernel (cooperative launch).  query: out[0] = own columns
// per warp, out[1] = co-resident CTAs per SM (nothing launched).
cudaError_t launch_prevrow_cb(int func, int variant, const FillParams& p, int nw, bool query, int* out,
                              cudaStream_t stream);
// Hierarchical-exchange prev-row kernel (prevrow_hx.cu; SCORE / LAST_ROW, one GPU, cooperative
// launch).  query: out[0] = own columns per CTA, out[1] = co-resident CTAs per SM, out[2] = outer
// halo HBO (edge pairs per CTA side).
cudaError_t launch_prevrow_hx(int func, int variant, const FillParams& p, bool query, int* out, cudaStream_t stream);
// Floyd-Steinberg lane-systolic knight kernel (fsk.cu): W warps per CTA, E extra lane lag.
cudaError_t launch_fsk(const FillParams& p, int W, int E, int R, int grid, cudaStream_t stream);
// Traceback of a LCS / Levenshtein / DTW table (traceback.cu): one thread, O(m + n).
cudaError_t launch_traceback(int func, const void* a, const void* b, const void* table, int64_t pitch, int64_t m,
                             int64_t n, int32_t* pi, int32_t* pj, int64_t* len, cudaStream_t s);
// Inverted-L kernel (invl.cu); mirror: read / write the grid with column j <-> W-1-j (the
// mInverted-L twin [L111]).
cudaError_t launch_invl(int func, const FillParams& p, int grid, bool mirror, cudaStream_t stream);
// TMA-staged inverted-L (no TABLE, 16-byte aligned grid, pitch % 4 == 0): cudaErrorNotSupported otherwise
cudaError_t launch_invl_tma(const FillParams& p, bool mirror, int sms, cudaStream_t stream);
// dst (cols x rows) = transpose of src (rows x cols), 32-bit elements, pitches in elements.
cudaError_t launch_transpose_i32(const int32_t* src, int64_t spitch, int32_t* dst, int64_t dpitch, int64_t rows,
                                 int64_t cols, cudaStream_t s);
// Packed 16x2 LCS kernel (lcs16.cu): P row pairs per lane (strips of 64P rows), lane lag E.
cudaError_t launch_lcs16(const FillParams& p, int P, int E, int grid, cudaStream_t stream);
bool lcs16_compiled(int P, int E);

// Per-kernel occupancy query (blocks per SM) for the chosen configuration.
int wavefront_blocks_per_sm(int func, int category, int rows_per_lane, int warps);
size_t wavefront_smem_bytes(int func, int category, int rows_per_lane, int warps);
bool wavefront_supported(int func, int category, int rows_per_lane, int warps);

}  // namespace lddp
