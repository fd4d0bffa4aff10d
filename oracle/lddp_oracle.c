/*
 * lddp_oracle.c -- plain, slow, obviously-correct CPU oracle for the LDDP-Plus table fill.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference leg may import, link or execute anything under oracle/.
 * The product path (paper_conf_ipps_kumark15_b200/) never touches this file, and this file
 * shares no source, header, table or constant with it.
 *
 * Citations: [Lnn] = /root/reference/PAPER.md line nn (Kumar & Kothapalli, IPDPSW 2015).
 *
 * What every function computes is the plain definition of the LDDP-Plus recurrence
 *     table[i][j] = f(table[i][j-1], table[i-1][j-1], table[i-1][j], table[i-1][j+1])
 * [L30 §I, general LDDP-Plus formula], [L94 §II], filled in row-major order.  Row-major order
 * is a valid topological order for every contributing set of Table I [L124-L142]: every
 * representative cell [L90] lies in row i-1 or at column j-1 of row i.  The paper's patterns
 * and phases only change WHEN a cell is evaluated, never WHAT it evaluates [L144], [L343-L344],
 * so no schedule appears here.
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math (no -march=native): floating point is
 * IEEE binary32 / binary64 scalar SSE, round-to-nearest-even, no FMA contraction, no FTZ.
 *
 * Readings where the paper is silent / garbled are listed in DESIGN.md §3 and repeated at
 * each function.  Parity pins for every function live in tests/test_oracle_pins.py.
 *
 * Output conventions (all optional, NULL = not requested):
 *   table     : the f-evaluated region, row-major with row pitch `pitch` (elements)
 *   last_row  : the f-evaluated region's bottom row
 *   last_col  : the f-evaluated region's right column
 * For LCS / Levenshtein / DTW the f-evaluated region is rows 1..m x cols 1..n of the
 * (m+1) x (n+1) table [L329]; row 0 / column 0 are the initialisation [L313].
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

/* ------------------------------------------------------------------------------------------
 * LCS -- Fig. 1(c) [L88] contributing set {L, UL, U}; Table I row "Y Y Y N" -> Anti-diagonal
 * [L139]; LCS is the Fig. 7 workload [L278].  The paper never prints the recurrence; this is
 * the textbook one (reading R1):
 *   L[i][0] = L[0][j] = 0
 *   L[i][j] = L[i-1][j-1] + 1                 if a[i-1] == b[j-1]
 *           = max(L[i-1][j], L[i][j-1])        otherwise
 * Returns L[m][n].
 * ---------------------------------------------------------------------------------------- */
int32_t oracle_lcs(const uint8_t* a, int64_t m, const uint8_t* b, int64_t n,
                   int32_t* table, int64_t pitch, int32_t* last_row, int32_t* last_col)
{
    if (m <= 0 || n <= 0) return 0;
    int32_t* prev = (int32_t*)calloc((size_t)(n + 1), sizeof(int32_t));   /* row i-1 */
    int32_t* cur  = (int32_t*)calloc((size_t)(n + 1), sizeof(int32_t));   /* row i   */
    for (int64_t i = 1; i <= m; ++i) {
        cur[0] = 0;                                         /* column 0 boundary */
        for (int64_t j = 1; j <= n; ++j) {
            if (a[i - 1] == b[j - 1]) {
                cur[j] = prev[j - 1] + 1;
            } else {
                cur[j] = prev[j] > cur[j - 1] ? prev[j] : cur[j - 1];
            }
        }
        if (table) memcpy(table + (i - 1) * pitch, cur + 1, (size_t)n * sizeof(int32_t));
        if (last_col) last_col[i - 1] = cur[n];
        int32_t* t = prev; prev = cur; cur = t;
    }
    if (last_row) memcpy(last_row, prev + 1, (size_t)n * sizeof(int32_t));
    int32_t score = prev[n];
    free(prev); free(cur);
    return score;
}

/* ------------------------------------------------------------------------------------------
 * Levenshtein distance -- §VI.A [L319-L329], Wagner-Fischer [19] [L405]:
 *   f(i,j) = max(i,j)                          if min(i,j) = 0
 *          = f(i-1,j-1)                        if a_i = b_j
 *          = 1 + min(f(i-1,j), f(i,j-1), f(i-1,j-1))   otherwise
 * The "min" is lost in the PDF extraction at [L325]; reading R7 restores it from
 * the definition "minimum number of single character edits" [L321] and [19].
 * Contributing set {L, UL, U} -> Anti-diagonal [L327].  Returns f(m,n).
 * ---------------------------------------------------------------------------------------- */
int32_t oracle_levenshtein(const uint8_t* a, int64_t m, const uint8_t* b, int64_t n,
                           int32_t* table, int64_t pitch, int32_t* last_row, int32_t* last_col)
{
    if (m <= 0) return (int32_t)(n > 0 ? n : 0);
    if (n <= 0) return (int32_t)m;
    int32_t* prev = (int32_t*)malloc((size_t)(n + 1) * sizeof(int32_t));
    int32_t* cur  = (int32_t*)malloc((size_t)(n + 1) * sizeof(int32_t));
    for (int64_t j = 0; j <= n; ++j) prev[j] = (int32_t)j;             /* max(0, j) */
    for (int64_t i = 1; i <= m; ++i) {
        cur[0] = (int32_t)i;                                           /* max(i, 0) */
        for (int64_t j = 1; j <= n; ++j) {
            if (a[i - 1] == b[j - 1]) {
                cur[j] = prev[j - 1];
            } else {
                int32_t best = prev[j];
                if (cur[j - 1] < best) best = cur[j - 1];
                if (prev[j - 1] < best) best = prev[j - 1];
                cur[j] = 1 + best;
            }
        }
        if (table) memcpy(table + (i - 1) * pitch, cur + 1, (size_t)n * sizeof(int32_t));
        if (last_col) last_col[i - 1] = cur[n];
        int32_t* t = prev; prev = cur; cur = t;
    }
    if (last_row) memcpy(last_row, prev + 1, (size_t)n * sizeof(int32_t));
    int32_t score = prev[n];
    free(prev); free(cur);
    return score;
}

/* ------------------------------------------------------------------------------------------
 * DTW -- named only as an LDDP-Plus example [L26 §I], reference [2] [L378]; the paper gives no
 * formula.  Reading R2: classic symmetric DTW, steps (1,0),(0,1),(1,1), unweighted,
 * no window, |x-y| local cost (BASELINE.json north star), binary32 storage and arithmetic
 * (north star: "fp32 DTW"):
 *   D[0][0] = 0, D[i][0] = D[0][j] = +inf (i,j >= 1)
 *   D[i][j] = |x[i-1] - y[j-1]| + min(min(D[i-1][j], D[i][j-1]), D[i-1][j-1])
 * Contributing set {L, UL, U} -> Anti-diagonal (Table I [L139]).  Returns D[m][n].
 * ---------------------------------------------------------------------------------------- */
float oracle_dtw(const float* x, int64_t m, const float* y, int64_t n,
                 float* table, int64_t pitch, float* last_row, float* last_col)
{
    if (m <= 0 && n <= 0) return 0.0f;
    if (m <= 0 || n <= 0) return INFINITY;
    float* prev = (float*)malloc((size_t)(n + 1) * sizeof(float));
    float* cur  = (float*)malloc((size_t)(n + 1) * sizeof(float));
    prev[0] = 0.0f;
    for (int64_t j = 1; j <= n; ++j) prev[j] = INFINITY;
    for (int64_t i = 1; i <= m; ++i) {
        cur[0] = INFINITY;
        for (int64_t j = 1; j <= n; ++j) {
            float cost = fabsf(x[i - 1] - y[j - 1]);
            float best = fminf(fminf(prev[j], cur[j - 1]), prev[j - 1]);
            cur[j] = cost + best;
        }
        if (table) memcpy(table + (i - 1) * pitch, cur + 1, (size_t)n * sizeof(float));
        if (last_col) last_col[i - 1] = cur[n];
        float* t = prev; prev = cur; cur = t;
    }
    if (last_row) memcpy(last_row, prev + 1, (size_t)n * sizeof(float));
    float score = prev[n];
    free(prev); free(cur);
    return score;
}

/* Same DTW definition in binary64 (used only to measure the binary32 rounding error). */
double oracle_dtw_f64(const double* x, int64_t m, const double* y, int64_t n)
{
    if (m <= 0 && n <= 0) return 0.0;
    if (m <= 0 || n <= 0) return INFINITY;
    double* prev = (double*)malloc((size_t)(n + 1) * sizeof(double));
    double* cur  = (double*)malloc((size_t)(n + 1) * sizeof(double));
    prev[0] = 0.0;
    for (int64_t j = 1; j <= n; ++j) prev[j] = INFINITY;
    for (int64_t i = 1; i <= m; ++i) {
        cur[0] = INFINITY;
        for (int64_t j = 1; j <= n; ++j) {
            double cost = fabs(x[i - 1] - y[j - 1]);
            double best = fmin(fmin(prev[j], cur[j - 1]), prev[j - 1]);
            cur[j] = cost + best;
        }
        double* t = prev; prev = cur; cur = t;
    }
    double score = prev[n];
    free(prev); free(cur);
    return score;
}

/* ------------------------------------------------------------------------------------------
 * Floyd-Steinberg dithering -- §VI.B [L341], Fig. 11 [L339], Floyd & Steinberg [12] [L397].
 * Textbook PUSH form, raster scan (left to right on every row):
 *   old = buf[i][j];  new = old >= 128 ? 255 : 0;  out[i][j] = new;  e = old - new;
 *   buf[i][j+1]   += e * 7/16      ("forwarded to cell_{i,j+1}")
 *   buf[i+1][j-1] += e * 3/16      ("cell_{i+1,j-1}")
 *   buf[i+1][j]   += e * 5/16      ("cell_{i+1,j}")
 *   buf[i+1][j+1] += e * 1/16      ("cell_{i+1,j+1}")        [L341]
 * Readings (R3-R5): threshold 128 with ties to 255; the error is taken from the
 * error-adjusted value (standard FS [12]; only this makes the scheduling constraint
 * [L343-L344] meaningful); binary32 arithmetic, each += is one rounded product (k/16 is exact)
 * then one rounded add, no FMA (north star: "fmad disabled and the oracle's operation order");
 * errors leaving the image are dropped; no clamping of buf.
 * Optional `err` receives e for every pixel (for the intensity-conservation pin).
 * ---------------------------------------------------------------------------------------- */
void oracle_fs(const uint8_t* in, int64_t H, int64_t W, uint8_t* out, float* err)
{
    if (H <= 0 || W <= 0) return;
    float* buf = (float*)malloc((size_t)(H * W) * sizeof(float));
    for (int64_t k = 0; k < H * W; ++k) buf[k] = (float)in[k];
    const float w7 = 7.0f / 16.0f, w3 = 3.0f / 16.0f, w5 = 5.0f / 16.0f, w1 = 1.0f / 16.0f;
    for (int64_t i = 0; i < H; ++i) {
        for (int64_t j = 0; j < W; ++j) {
            float old = buf[i * W + j];
            float nw = (old >= 128.0f) ? 255.0f : 0.0f;
            out[i * W + j] = (uint8_t)nw;
            float e = old - nw;
            if (err) err[i * W + j] = e;
            if (j + 1 < W) buf[i * W + j + 1] += e * w7;
            if (i + 1 < H) {
                if (j > 0) buf[(i + 1) * W + j - 1] += e * w3;
                buf[(i + 1) * W + j] += e * w5;
                if (j + 1 < W) buf[(i + 1) * W + j + 1] += e * w1;
            }
        }
    }
    free(buf);
}

/* ------------------------------------------------------------------------------------------
 * Checkerboard minimum path -- §VI.C [L350-L367].  c is H x W int32.
 *   f[0][j] = c[0][j]                                                 ("if i = 1" [L360])
 *   f[i][j] = c[i][j] + min{ f[i-1][k] : k in {j-1, j, j+1} and 0 <= k < W }
 * Readings (R6): three-term min (the extraction at [L362] shows two terms, [L365]
 * says three contributing cells); out-of-range neighbours are excluded ("inf if j<1 or j>n"
 * [L358]); 0-based indices.  Contributing set {UL, U, UR} -> Horizontal case-2 [L365].
 * Returns min_j f[H-1][j] (the shortest path cost to the last row [L352]).
 * ---------------------------------------------------------------------------------------- */
int32_t oracle_minpath3(const int32_t* c, int64_t H, int64_t W,
                        int32_t* table, int64_t pitch, int32_t* last_row)
{
    if (H <= 0 || W <= 0) return 0;
    int32_t* prev = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t* cur  = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    for (int64_t j = 0; j < W; ++j) prev[j] = c[j];
    if (table) memcpy(table, prev, (size_t)W * sizeof(int32_t));
    for (int64_t i = 1; i < H; ++i) {
        for (int64_t j = 0; j < W; ++j) {
            int32_t best = prev[j];
            if (j - 1 >= 0 && prev[j - 1] < best) best = prev[j - 1];
            if (j + 1 < W && prev[j + 1] < best) best = prev[j + 1];
            cur[j] = c[i * W + j] + best;
        }
        if (table) memcpy(table + i * pitch, cur, (size_t)W * sizeof(int32_t));
        int32_t* t = prev; prev = cur; cur = t;
    }
    if (last_row) memcpy(last_row, prev, (size_t)W * sizeof(int32_t));
    int32_t best = prev[0];
    for (int64_t j = 1; j < W; ++j) if (prev[j] < best) best = prev[j];
    free(prev); free(cur);
    return best;
}

/* ------------------------------------------------------------------------------------------
 * Horizontal case-1 synthetic f -- §V.B [L298], Fig. 9 [L306]:
 *   f(i,j) = min(f(i-1,j-1), f(i-1,j)) + c
 * Readings (R8): row 0 is the user initialisation init[0][.] [L313]; at j = 0 the
 * absent UL is excluded (only f(i-1,0)).  Contributing set {UL, U} -> Horizontal (Table I
 * [L131]).  Returns min_j f[H-1][j].
 * ---------------------------------------------------------------------------------------- */
int32_t oracle_min2plus(const int32_t* init, int64_t H, int64_t W, int32_t cst,
                        int32_t* table, int64_t pitch, int32_t* last_row)
{
    if (H <= 0 || W <= 0) return 0;
    int32_t* prev = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t* cur  = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    for (int64_t j = 0; j < W; ++j) prev[j] = init[j];
    if (table) memcpy(table, prev, (size_t)W * sizeof(int32_t));
    for (int64_t i = 1; i < H; ++i) {
        for (int64_t j = 0; j < W; ++j) {
            int32_t best = prev[j];
            if (j - 1 >= 0 && prev[j - 1] < best) best = prev[j - 1];
            cur[j] = best + cst;
        }
        if (table) memcpy(table + i * pitch, cur, (size_t)W * sizeof(int32_t));
        int32_t* t = prev; prev = cur; cur = t;
    }
    if (last_row) memcpy(last_row, prev, (size_t)W * sizeof(int32_t));
    int32_t best = prev[0];
    for (int64_t j = 1; j < W; ++j) if (prev[j] < best) best = prev[j];
    free(prev); free(cur);
    return best;
}

/* ------------------------------------------------------------------------------------------
 * Inverted-L synthetic f -- §V.B [L298], Fig. 8 [L286]:
 *   f(i,j) = max(cell_{i,j}, f(i-1,j-1)) + c
 * Readings (R9): cell_{i,j} is the cell's user-initialised value init[i][j] [L313];
 * row 0 and column 0 are init (boundary).  Contributing set {UL} -> Inverted-L (Table I
 * [L129], [L203]).
 * ---------------------------------------------------------------------------------------- */
void oracle_diagmaxplus(const int32_t* init, int64_t H, int64_t W, int32_t cst,
                        int32_t* table, int64_t pitch, int32_t* last_row, int32_t* last_col)
{
    if (H <= 0 || W <= 0) return;
    int32_t* prev = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t* cur  = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    for (int64_t j = 0; j < W; ++j) prev[j] = init[j];
    if (table) memcpy(table, prev, (size_t)W * sizeof(int32_t));
    if (last_col) last_col[0] = prev[W - 1];
    for (int64_t i = 1; i < H; ++i) {
        cur[0] = init[i * W];
        for (int64_t j = 1; j < W; ++j) {
            int32_t v = init[i * W + j];
            if (prev[j - 1] > v) v = prev[j - 1];
            cur[j] = v + cst;
        }
        if (table) memcpy(table + i * pitch, cur, (size_t)W * sizeof(int32_t));
        if (last_col) last_col[i] = cur[W - 1];
        int32_t* t = prev; prev = cur; cur = t;
    }
    if (last_row) memcpy(last_row, prev, (size_t)W * sizeof(int32_t));
    free(prev); free(cur);
}

/* ------------------------------------------------------------------------------------------
 * The two symmetric twins of Table I [L109-L113] ("Vertical is the transpose of Horizontal,
 * mInverted-L the mirror of Inverted-L" [L111]), instantiated with the synthetic f's of §V.B
 * [L298] so that every one of the six patterns has a compiled-in f (reading R15).
 *
 * MIN2_PLUS_V (Vertical, contributing set {L, UL}, Table I [L137]):
 *   f(i,0) = init[i][0] (column 0 is the boundary);  f(0,j) = f(0,j-1) + c (only L exists);
 *   f(i,j) = min(f(i,j-1), f(i-1,j-1)) + c.
 * Outputs: last_col (the right column, where the column sweep ends) and its minimum.
 * ---------------------------------------------------------------------------------------- */
int32_t oracle_min2plus_v(const int32_t* init, int64_t H, int64_t W, int32_t cst,
                          int32_t* table, int64_t pitch, int32_t* last_col)
{
    if (H <= 0 || W <= 0) return 0;
    int32_t* prev = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t* cur  = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t best = 0;
    for (int64_t i = 0; i < H; ++i) {
        for (int64_t j = 0; j < W; ++j) {
            if (j == 0) {
                cur[j] = init[i * W];
            } else {
                int32_t m = cur[j - 1];                           /* L  */
                if (i > 0 && prev[j - 1] < m) m = prev[j - 1];    /* UL */
                cur[j] = m + cst;
            }
        }
        if (table) memcpy(table + i * pitch, cur, (size_t)W * sizeof(int32_t));
        if (last_col) last_col[i] = cur[W - 1];
        if (i == 0 || cur[W - 1] < best) best = cur[W - 1];
        int32_t* t = prev; prev = cur; cur = t;
    }
    free(prev); free(cur);
    return best;
}

/* ANTIDIAG_MAXPLUS (mInverted-L, contributing set {UR}, Table I [L126]):
 *   f(i,j) = init[i][j] on row 0 and on column W-1 (the boundary);
 *   f(i,j) = max(init[i][j], f(i-1,j+1)) + c.
 * Its chains run down-left and end on the last row or on column 0.  Outputs: last_row and
 * first_col (column 0, where the chains end). */
void oracle_antidiag_maxplus(const int32_t* init, int64_t H, int64_t W, int32_t cst,
                             int32_t* table, int64_t pitch, int32_t* last_row, int32_t* first_col)
{
    if (H <= 0 || W <= 0) return;
    int32_t* prev = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t* cur  = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    for (int64_t i = 0; i < H; ++i) {
        for (int64_t j = 0; j < W; ++j) {
            int32_t v = init[i * W + j];
            if (i > 0 && j < W - 1) {
                if (prev[j + 1] > v) v = prev[j + 1];             /* UR */
                v += cst;
            }
            cur[j] = v;
        }
        if (table) memcpy(table + i * pitch, cur, (size_t)W * sizeof(int32_t));
        if (first_col) first_col[i] = cur[0];
        int32_t* t = prev; prev = cur; cur = t;
    }
    if (last_row) memcpy(last_row, prev, (size_t)W * sizeof(int32_t));
    free(prev); free(cur);
}
