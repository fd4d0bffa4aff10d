/*
 * lddp.h -- C ABI of the B200-native LDDP-Plus table fill (liblddp.so).
 *
 * The method (Kumar & Kothapalli, "A Novel Heterogeneous Framework for Local Dependency
 * Dynamic Programming Problems", IPDPSW 2015; citations [Lnn] = /root/reference/PAPER.md line nn):
 *
 *     table[i][j] = f(table[i][j-1], table[i-1][j-1], table[i-1][j], table[i-1][j+1])
 *                                                        [L30 §I formula], [L94 §II]
 *
 * The four neighbours are the paper's representative set RS(i,j) [L90]: L = cell_{i,j-1},
 * UL = cell_{i-1,j-1}, U = cell_{i-1,j}, UR = cell_{i-1,j+1}.  The subset f actually reads is
 * its contributing set [L90-L94]; Table I [L124-L142] maps the 15 contributing sets to six
 * patterns, folded by symmetry to four [L111]: these are the dependency categories below.
 * The user supplies f and the initialisation [L300-L313]; in this build f is compiled in
 * (lddp_func) and its initialisation is implied by f.
 *
 * Conventions
 *  - Every call returns lddp_status (LDDP_OK = 0).  Nothing throws or aborts across the ABI;
 *    the failing call's message is available from lddp_last_error_message() (thread-local).
 *  - All buffer pointers in lddp_inputs / lddp_outputs and the workspace are DEVICE pointers
 *    owned by the caller (except lddp_fill_host, which takes host pointers).  They must stay
 *    valid until the enqueued work completes.  Inputs are never written.
 *  - lddp_fill / lddp_fill_multi only ENQUEUE on the given cudaStream_t (passed as void*); they
 *    never synchronise.  Argument and shape errors are reported synchronously; a device-side
 *    watchdog timeout is reported by lddp_status_check() after the stream completes.
 *  - A plan is immutable after creation and owns only host metadata (plus, if the caller
 *    never supplies one, a lazily allocated default workspace).  Concurrent fills with one
 *    plan need distinct workspaces and streams.
 *  - Element types: LCS / Levenshtein / min-path / synthetic f's use int32; DTW uses IEEE
 *    binary32; Floyd-Steinberg reads and writes uint8 pixels (errors are binary32 internally).
 *  - The caller guarantees no int32 overflow (path sums < 2^31).
 */
#ifndef LDDP_H_
#define LDDP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LDDP_ABI_VERSION 2

typedef enum {
    LDDP_OK = 0,
    LDDP_ERR_INVALID_ARG = 1,       /* NULL pointer, bad enum, missing required buffer        */
    LDDP_ERR_SHAPE = 2,             /* negative size, or a size the f / category cannot take   */
    LDDP_ERR_CATEGORY_MISMATCH = 3, /* the category's schedule does not order f's contributing
                                       set (Table I [L124-L142] + Fig. 2 [L117-L122])           */
    LDDP_ERR_UNSUPPORTED = 4,       /* valid request this build does not implement            */
    LDDP_ERR_OUT_OF_MEMORY = 5,
    LDDP_ERR_CUDA = 6,              /* a CUDA runtime call failed (message has the detail)     */
    LDDP_ERR_COMM = 7,              /* multi-GPU window / IPC failure                          */
    LDDP_ERR_TIMEOUT = 8,           /* device watchdog: a dependency wait exceeded the budget  */
    LDDP_ERR_INTERNAL = 9
} lddp_status;

/* Dependency categories = the paper's four distinct patterns [L109-L111], Fig. 2 [L117-L122].
 * The iteration number of cell (i,j) (0-based) is the schedule each category's kernel follows
 * at tile granularity. */
typedef enum {
    LDDP_CAT_PREV_ROW = 0,      /* "Horizontal" [L180-L195]: t = i.  Masks within {UL,U,UR}      */
    LDDP_CAT_ANTI_DIAGONAL = 1, /* [L148-L168]: t = i + j.  Masks within {L,UL,U}                */
    LDDP_CAT_KNIGHT_MOVE = 2,   /* "all-four-neighbour skewed" [L217-L241]: t = 2i + j.  Any mask */
    LDDP_CAT_INVERTED_L = 3,    /* the remaining pattern [L197-L215]: t = min(i,j).  Mask {UL}   */
    /* The two symmetric twins of Table I [L109-L113]: "Vertical is the transpose of Horizontal,
     * mInverted-L the mirror of Inverted-L" [L111].  They run on the kernels of their twins. */
    LDDP_CAT_VERTICAL = 4,      /* t = j (column sweep).  Mask within {L,UL}.  Transpose (a tiled
                                   transpose kernel into the workspace) + the prev-row kernel   */
    LDDP_CAT_MINVERTED_L = 5    /* t = min(i, W-1-j).  Mask {UR}.  The inverted-L kernel reading
                                   the grid mirrored (column j <-> W-1-j), no copy              */
} lddp_category;

/* The six patterns of Table I (lddp_classify reports the paper's pattern for a mask). */
typedef enum {
    LDDP_PAT_HORIZONTAL = 0,
    LDDP_PAT_ANTI_DIAGONAL = 1,
    LDDP_PAT_KNIGHT_MOVE = 2,
    LDDP_PAT_INVERTED_L = 3,
    LDDP_PAT_VERTICAL = 4,      /* symmetric twin of Horizontal [L111] (transpose)               */
    LDDP_PAT_MINVERTED_L = 5    /* symmetric twin of Inverted-L [L111] (mirror)                  */
} lddp_pattern;

/* Contributing-set bits over RS(i,j) [L90]. */
#define LDDP_NB_L  1u   /* cell_{i,j-1}   */
#define LDDP_NB_UL 2u   /* cell_{i-1,j-1} */
#define LDDP_NB_U  4u   /* cell_{i-1,j}   */
#define LDDP_NB_UR 8u   /* cell_{i-1,j+1} */

/* Compiled-in cell functions.  rows x cols is always the f-evaluated region.
 *  LCS          [L88] Fig.1(c): region = rows 1..m, cols 1..n of the (m+1)x(n+1) table; row 0 /
 *               col 0 = 0.  inputs.a = uint8[m], inputs.b = uint8[n].  mask {L,UL,U}.
 *  DTW          [L26] + reading R2: D[0][0]=0, D[i][0]=D[0][j]=+inf; cell = |x_i - y_j| +
 *               min(U, L, UL) in binary32.  inputs.a = float[m], inputs.b = float[n].  {L,UL,U}.
 *  FS_DITHER    [L341-L344] Floyd-Steinberg, pull form of the raster push form (threshold 128,
 *               ties to 255, binary32, no FMA).  inputs.grid = uint8 HxW; outputs.table =
 *               uint8 HxW output image (required).  mask {L,UL,U,UR}.
 *  MIN_PATH3    [L350-L367] checkerboard: f[0][j] = c[0][j]; f[i][j] = c[i][j] + min of the
 *               in-range {UL,U,UR}.  inputs.grid = int32 HxW costs.  mask {UL,U,UR}.
 *  DIAG_MAXPLUS [L298] f = max(init[i][j], f(i-1,j-1)) + c; row 0 / col 0 = init.  {UL}.
 *  MIN2_PLUS    [L298] f = min(f(i-1,j-1), f(i-1,j)) + c; row 0 = init; j=0 uses U only. {UL,U}.
 *  LEVENSHTEIN  [L319-L329] f = max(i,j) if min(i,j)=0; UL if a_i=b_j; else 1+min(U,L,UL).
 *               Same layout as LCS.  mask {L,UL,U}.
 *  MIN2_PLUS_V  the Vertical twin of MIN2_PLUS (reading R15): f = min(L, UL) + c; column 0 =
 *               init; row 0 uses L only.  SCORE = min of the last column.  mask {L,UL};
 *               category VERTICAL only.
 *  ANTIDIAG_MAXPLUS  the mInverted-L twin of DIAG_MAXPLUS (R15): f = max(init, UR) + c; row 0
 *               and column W-1 = init.  LAST_COL = column 0 (where its chains end).  mask {UR};
 *               category MINVERTED_L only.                                                      */
typedef enum {
    LDDP_F_LCS = 0,
    LDDP_F_DTW = 1,
    LDDP_F_FS_DITHER = 2,
    LDDP_F_MIN_PATH3 = 3,
    LDDP_F_DIAG_MAXPLUS = 4,
    LDDP_F_MIN2_PLUS = 5,
    LDDP_F_LEVENSHTEIN = 6,
    LDDP_F_MIN2_PLUS_V = 7,
    LDDP_F_ANTIDIAG_MAXPLUS = 8
} lddp_func;

/* Requested outputs (bitmask). */
#define LDDP_OUT_SCORE    1u  /* LCS/Lev int32 L[m][n]; DTW float D[m][n]; MIN_PATH3/MIN2_PLUS
                                 int32 min of the last row.  Not valid for FS / DIAG_MAXPLUS.   */
#define LDDP_OUT_LAST_ROW 2u  /* bottom row of the region: cols elements                        */
#define LDDP_OUT_LAST_COL 4u  /* right column of the region: rows elements (anti-diagonal,
                                 knight-move, inverted-L and vertical categories; column 0 for
                                 ANTIDIAG_MAXPLUS).  Not produced by the prev-row category.      */
#define LDDP_OUT_TABLE    8u  /* whole region, row-major, pitch outputs.table_pitch elements.
                                 Always required (and implied) for FS_DITHER (output image).    */

typedef struct {
    int64_t rows;            /* m (LCS/Lev/DTW) or H                                            */
    int64_t cols;            /* n (LCS/Lev/DTW) or W                                            */
    int32_t category;        /* lddp_category                                                   */
    int32_t func;            /* lddp_func                                                       */
    uint32_t outputs;        /* LDDP_OUT_* bitmask                                              */
    int32_t param_c;         /* constant c of DIAG_MAXPLUS / MIN2_PLUS [L298]                   */
    int32_t device;          /* CUDA device ordinal the plan is bound to                        */
    int32_t tile_rows;       /* tuning: rows per lane (anti-diagonal / knight), 0 = auto        */
    int32_t tile_warps;      /* tuning: compute warps per CTA, 0 = auto                         */
    int32_t band_rows;       /* tuning, prev-row category: trapezoid band height HB (rows between
                                two halo exchanges of the column-block kernel prevrow_cb): 16,
                                32, 48 or 64 (else LDDP_ERR_UNSUPPORTED); 0 = auto (SCORE /
                                LAST_ROW / TABLE fills, also lddp_fill_multi: the hierarchical-
                                exchange kernel, inner halos every 16 rows, CTA-edge halos
                                every 96; TABLE pitches that are not multiples of 4, and
                                multi-GPU plans too narrow for one CTA strip per rank:
                                prevrow_cb with HB = 32)                                        */
    int32_t grid_ctas;       /* tuning: persistent grid size, 0 = auto (SMs x occupancy)        */
    int32_t batch;           /* FS_DITHER only: number of independent images stacked along the
                                rows (image b = rows [b*rows, (b+1)*rows) of inputs.grid and of
                                outputs.table, same pitches); 0 or 1 = one image.  All images
                                are filled by ONE launch whose warps claim (strip, image) pairs
                                strip-major, so the images' pipelines run concurrently
                                (batched FS, image-parallel [L335-L348], reading R21).
                                lddp_fill_multi gives rank g images [g*B/P, (g+1)*B/P).     */
    int32_t reserved[2];     /* must be 0                                                       */
} lddp_desc;

typedef struct {
    const void* a;           /* LCS/Lev: const uint8_t[rows]; DTW: const float[rows]            */
    const void* b;           /* LCS/Lev: const uint8_t[cols]; DTW: const float[cols]            */
    const void* grid;        /* FS: const uint8_t, MIN_PATH3/DIAG_MAXPLUS/MIN2_PLUS: const
                                int32_t; rows x cols, row pitch grid_pitch elements             */
    int64_t grid_pitch;      /* elements; >= cols.  FS additionally needs pitch % 4 == 0 and a
                                4-byte aligned base (word-wide pixel loads).  Fast paths, chosen
                                per fill, fall back to the generic kernels otherwise:
                                - FS (fsk.cu): cols % 16 == 0, grid and table pitches multiples
                                  of 16 bytes, 16-byte aligned bases;
                                - prev-row (prevrow_hx.cu / prevrow_cb.cu): 32-bit grid,
                                  cols % 4 == 0, pitch % 4 == 0, 16-byte aligned base, and the
                                  column blocks co-resident on the device (checked at plan
                                  time; prevrow_hx also rows < 2^30, pitch < 2^29)           */
} lddp_inputs;

typedef struct {
    void* score;             /* 1 element (int32 or float), or NULL                             */
    void* last_row;          /* cols elements, or NULL                                          */
    void* last_col;          /* rows elements, or NULL                                          */
    void* table;             /* rows x cols, pitch table_pitch; FS: uint8 image (pitch % 4 == 0) */
    int64_t table_pitch;     /* elements                                                        */
} lddp_outputs;

typedef struct lddp_plan_s* lddp_plan_t;
typedef struct lddp_comm_s* lddp_comm_t;

/* ---- host-only queries (no GPU needed) --------------------------------------------------- */
int32_t lddp_abi_version(void);
const char* lddp_status_string(lddp_status s);
const char* lddp_last_error_message(void);              /* thread-local, of the last failure */
/* Contributing set of a compiled-in f (LDDP_NB_* bits). */
lddp_status lddp_func_mask(int32_t func, uint32_t* mask);
/* Table I [L124-L142]: the paper's pattern for a non-empty contributing set (1..15). */
lddp_status lddp_classify(uint32_t mask, int32_t* pattern);
/* 1 if the category's schedule (Fig. 2 [L117-L122]) strictly orders every dependency in mask
 * (a more general category is always allowed, e.g. Knight-Move covers all 15 sets). */
lddp_status lddp_category_covers(int32_t category, uint32_t mask, int32_t* covers);

/* ---- plans --------------------------------------------------------------------------------
 * lddp_plan validates the (f, category, shape, outputs) request and fixes the launch geometry
 * (needs the CUDA device to query its SM count).  Errors: INVALID_ARG, SHAPE,
 * CATEGORY_MISMATCH (category does not cover f's mask), UNSUPPORTED, CUDA. */
lddp_status lddp_plan(const lddp_desc* desc, lddp_plan_t* plan);
lddp_status lddp_plan_destroy(lddp_plan_t plan);
/* Bytes of device workspace lddp_fill needs (0 is possible). */
lddp_status lddp_plan_workspace_size(lddp_plan_t plan, size_t* bytes);
/* JSON description of the chosen geometry (kernel, grid, block, rows per lane, ...). */
lddp_status lddp_plan_describe(lddp_plan_t plan, char* buf, size_t len);
/* Zero a caller-owned workspace (required once before its first use, and after a TIMEOUT). */
lddp_status lddp_workspace_init(lddp_plan_t plan, void* workspace, void* stream);

/* ---- the fill -------------------------------------------------------------------------------
 * Enqueue one dependency-ordered fill of the table on `stream` (cudaStream_t; NULL = default
 * stream).  workspace: device buffer of lddp_plan_workspace_size bytes, zeroed once with
 * lddp_workspace_init; NULL = the plan's own workspace.  One persistent kernel launch (per
 * category) -- no launch per diagonal [L150]. */
lddp_status lddp_fill(lddp_plan_t plan, const lddp_inputs* in, const lddp_outputs* out,
                      void* workspace, void* stream);
/* Same fill from HOST buffers: copies inputs host->device, fills, copies the requested outputs
 * device->host and synchronises `stream`.  Device staging buffers are owned by the plan. */
lddp_status lddp_fill_host(lddp_plan_t plan, const lddp_inputs* host_in,
                           const lddp_outputs* host_out, void* stream);
/* Traceback of a LCS / Levenshtein / DTW table written by lddp_fill with
 * LDDP_OUT_TABLE (same plan; T[i-1][j-1] = D[i][j], row / column 0 implied by f's boundary).
 * One device thread walks from DP cell (m, n) towards the boundary and writes the visited cells
 * (i, j), 1 <= i <= m, 1 <= j <= n, to path_i / path_j (device int32 arrays of capacity
 * m + n, caller-owned) and their count to *path_len (device int64).  Rules (R14):
 *   LCS   a_i == b_j -> diagonal; else up if D[i-1][j] >= D[i][j-1], else left (CLRS);
 *   Lev   diagonal on a match with equal cost, else the first of substitution, deletion,
 *         insertion that reproduces D[i][j];
 *   DTW   argmin of (UL, U, L), ties in that order, ends at (1, 1).
 * in->a / in->b: the fill's device inputs.  Enqueues on `stream`; errors: INVALID_ARG,
 * UNSUPPORTED (another f), CUDA. */
lddp_status lddp_traceback(lddp_plan_t plan, const lddp_inputs* in, const void* table, int64_t table_pitch,
                           int32_t* path_i, int32_t* path_j, int64_t* path_len, void* stream);
/* Synchronise `stream` and read the workspace's device status word (watchdog). */
lddp_status lddp_status_check(lddp_plan_t plan, void* workspace, void* stream);

/* ---- multi-GPU column strips (one process per GPU) -------------------------------------------
 * Rank g of P owns columns [floor(g*cols/P), floor((g+1)*cols/P)) of every row
 * (lddp_multi_partition).  Each rank's persistent kernel stores the right column of every
 * finished row strip straight into rank g+1's receive window over NVLink (peer stores + a
 * system-scope release flag per strip: the one-way boundary transfer of Table II's
 * anti-diagonal row [L265-L274], [L164]) and reads rank g-1's column from its own window.
 * Supported categories:
 *   anti-diagonal (LCS, Levenshtein, DTW): column strips, one-way boundary transfer (above);
 *   previous-row (min-path, min2plus; cols % 4 == 0): column strips made of whole column blocks
 *     of the column-block kernel (lddp_plan_partition); every HB-row band the strip's outer
 *     blocks store their HB edge columns into the neighbour ranks' windows as tagged (value,
 *     fill epoch | band) pairs and read the neighbours' edges from their own window -- the
 *     two-way trapezoid halo of Table II case 2 [L265-L274], [L193-L195].  Window halo region:
 *     [from g-1: 8 slots][from g+1: 8 slots] x 64 pairs, slot = (fill parity, band mod 4).
 *     Every rank's kernel must be resident at once (they exchange every band).  Rank g writes
 *     last_row / table columns [c0, c1) and score = the minimum of ITS last-row columns (the
 *     global score is the minimum over ranks);
 *   inverted-L / mInverted-L: diagonal shares d = j - i in [lo, hi) holding ~1/P of the cells
 *     (every chain independent [L203]): no exchange; rank g writes its chains' cells and ends.
 *
 * Window of rank g (device memory of rank g), two slots selected by fill parity so that fill
 * k+1 can start on rank g-1 while rank g is still reading fill k:
 *   ack[2][S]       written by rank g+1: fill epoch whose strip s it has finished reading
 *   flag[2][S]      written by rank g-1: (epoch << 32) | 1 once strip s's column is in
 *   value[2][m + 1] written by rank g-1: its right column, index i + 1 for row i
 * A producer reuses slot k & 1 for strip s only after the consumer acknowledged fill k-2 for
 * strips s and s+1 (strip s+1 also reads strip s's last row); a consumer accepts a flag only if it
 * equals this fill's epoch.  Every wait is bounded by the device watchdog (LDDP_ERR_TIMEOUT).
 *   lddp_comm_create   allocates this rank's window on the plan's device (zeroed).
 *   lddp_comm_handle   exports it (CUDA IPC handle, LDDP_COMM_HANDLE_BYTES).
 *   lddp_comm_connect  opens rank g+1's and rank g-1's windows from their handles (NULL at the
 *                      ends of the chain).  Handles travel over any process group (the
 *                      torch.distributed gloo / NCCL object collectives in bench.py and tests).
 *   lddp_comm_connect_local   in-process alternative (ranks on the same or peer devices).
 * lddp_fill_multi: every rank calls it once per fill, in the same order (the k-th call on each
 * rank is fill k), with the whole a / b (rows / cols of the full problem) and full-size output
 * buffers; rank g writes last_row[c0:c1) and, on the last rank only, score and last_col.  Fills
 * only enqueue: ranks may run ahead of each other by up to one fill. */
#define LDDP_COMM_HANDLE_BYTES 64
/* Columns [c0, c1) of rank `rank` of `nranks` for a problem with `cols` columns (host only). */
lddp_status lddp_multi_partition(int64_t cols, int32_t nranks, int32_t rank, int64_t* c0, int64_t* c1);
/* The share of rank `rank` of `nranks` in lddp_fill_multi for this plan: columns [lo, hi) for
 * column strips (anti-diagonal: lddp_multi_partition; prev-row: whole column blocks), diagonals
 * d = j - i in [lo, hi) for inverted-L shares.  Host only; errors: INVALID_ARG. */
lddp_status lddp_plan_partition(lddp_plan_t plan, int32_t nranks, int32_t rank, int64_t* lo, int64_t* hi);
lddp_status lddp_comm_create(lddp_plan_t plan, int32_t nranks, int32_t rank, lddp_comm_t* comm);
lddp_status lddp_comm_handle(lddp_comm_t comm, uint8_t handle[LDDP_COMM_HANDLE_BYTES]);
lddp_status lddp_comm_connect(lddp_comm_t comm, const uint8_t* next_handle, const uint8_t* prev_handle);
lddp_status lddp_comm_connect_local(lddp_comm_t comm, lddp_comm_t next, lddp_comm_t prev);
lddp_status lddp_comm_destroy(lddp_comm_t comm);
lddp_status lddp_fill_multi(lddp_plan_t plan, const lddp_inputs* in, const lddp_outputs* out,
                            void* workspace, lddp_comm_t comm, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* LDDP_H_ */
