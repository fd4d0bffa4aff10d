"""CPU oracle for the LDDP-Plus table fill (ctypes wrapper over oracle/lddp_oracle.c).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` leg may import this package.  The product package
``paper_conf_ipps_kumark15_b200`` never imports it, and it imports nothing from the product.

Every function is the plain row-major definition of one compiled-in ``f`` (see the C file for
the paper passages each follows).  Inputs are numpy arrays; outputs are numpy arrays / scalars.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lddp_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liblddp_oracle.so")

# -ffp-contract=off: GCC's GNU-mode default is -ffp-contract=fast (FMA contraction); the
# oracle's binary32 operation order must be exactly the written one.  No -march=native.
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile liblddp_oracle.so next to the source (idempotent)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        i64, p = ctypes.c_int64, ctypes.c_void_p
        lib.oracle_lcs.restype = ctypes.c_int32
        lib.oracle_lcs.argtypes = [p, i64, p, i64, p, i64, p, p]
        lib.oracle_levenshtein.restype = ctypes.c_int32
        lib.oracle_levenshtein.argtypes = [p, i64, p, i64, p, i64, p, p]
        lib.oracle_dtw.restype = ctypes.c_float
        lib.oracle_dtw.argtypes = [p, i64, p, i64, p, i64, p, p]
        lib.oracle_dtw_f64.restype = ctypes.c_double
        lib.oracle_dtw_f64.argtypes = [p, i64, p, i64]
        lib.oracle_fs.restype = None
        lib.oracle_fs.argtypes = [p, i64, i64, p, p]
        lib.oracle_minpath3.restype = ctypes.c_int32
        lib.oracle_minpath3.argtypes = [p, i64, i64, p, i64, p]
        lib.oracle_min2plus.restype = ctypes.c_int32
        lib.oracle_min2plus.argtypes = [p, i64, i64, ctypes.c_int32, p, i64, p]
        lib.oracle_diagmaxplus.restype = None
        lib.oracle_diagmaxplus.argtypes = [p, i64, i64, ctypes.c_int32, p, i64, p, p]
        lib.oracle_min2plus_v.restype = ctypes.c_int32
        lib.oracle_min2plus_v.argtypes = [p, i64, i64, ctypes.c_int32, p, i64, p]
        lib.oracle_antidiag_maxplus.restype = None
        lib.oracle_antidiag_maxplus.argtypes = [p, i64, i64, ctypes.c_int32, p, i64, p, p]
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dtype):
    return np.ascontiguousarray(np.asarray(a, dtype=dtype))


class Result(dict):
    """score / last_row / last_col / table, whichever were requested."""

    __getattr__ = dict.get


def _seq_fill(fn, a, b, dtype_in, dtype_out, table, rows):
    a = _c(a, dtype_in)
    b = _c(b, dtype_in)
    m, n = len(a), len(b)
    last_row = np.empty(n, dtype_out) if rows else None
    last_col = np.empty(m, dtype_out) if rows else None
    tab = np.empty((m, n), dtype_out) if table else None
    score = fn(_ptr(a), m, _ptr(b), n, _ptr(tab), n, _ptr(last_row), _ptr(last_col))
    return Result(score=score, last_row=last_row, last_col=last_col, table=tab)


def lcs(a, b, table: bool = False, rows: bool = True) -> Result:
    """LCS length table ([L88] Fig. 1(c), textbook recurrence); a, b: uint8 sequences."""
    return _seq_fill(_L().oracle_lcs, a, b, np.uint8, np.int32, table, rows)


def levenshtein(a, b, table: bool = False, rows: bool = True) -> Result:
    """Levenshtein distance table ([L319-L329] §VI.A)."""
    return _seq_fill(_L().oracle_levenshtein, a, b, np.uint8, np.int32, table, rows)


def dtw(x, y, table: bool = False, rows: bool = True) -> Result:
    """binary32 DTW table, |x-y| cost ([L26], reading R2)."""
    r = _seq_fill(_L().oracle_dtw, x, y, np.float32, np.float32, table, rows)
    r["score"] = np.float32(r["score"])
    return r


def dtw_f64(x, y) -> float:
    """The same DTW definition evaluated in binary64 (error reference for the fp32 path)."""
    x = _c(x, np.float64)
    y = _c(y, np.float64)
    return float(_L().oracle_dtw_f64(_ptr(x), len(x), _ptr(y), len(y)))


def fs(img, want_err: bool = False):
    """Floyd-Steinberg dithering, push form ([L341] §VI.B).  Returns out (uint8) [, err]."""
    img = _c(img, np.uint8)
    H, W = img.shape
    out = np.empty((H, W), np.uint8)
    err = np.empty((H, W), np.float32) if want_err else None
    _L().oracle_fs(_ptr(img), H, W, _ptr(out), _ptr(err))
    return (out, err) if want_err else out


def _grid_fill(fn, grid, extra, table, want_col=False):
    grid = _c(grid, np.int32)
    H, W = grid.shape
    tab = np.empty((H, W), np.int32) if table else None
    last_row = np.empty(W, np.int32)
    if want_col:
        last_col = np.empty(H, np.int32)
        fn(_ptr(grid), H, W, *extra, _ptr(tab), W, _ptr(last_row), _ptr(last_col))
        return Result(last_row=last_row, last_col=last_col, table=tab)
    score = fn(_ptr(grid), H, W, *extra, _ptr(tab), W, _ptr(last_row))
    return Result(score=score, last_row=last_row, table=tab)


def minpath3(cost, table: bool = False) -> Result:
    """Checkerboard min-path ([L350-L367] §VI.C), 3-term min."""
    return _grid_fill(_L().oracle_minpath3, cost, (), table)


def min2plus(init, c: int = 1, table: bool = False) -> Result:
    """Horizontal case-1 synthetic f = min(UL, U) + c ([L298] §V.B)."""
    return _grid_fill(_L().oracle_min2plus, init, (int(c),), table)


def diagmaxplus(init, c: int = 1, table: bool = False) -> Result:
    """Inverted-L synthetic f = max(init, UL) + c ([L298] §V.B)."""
    return _grid_fill(_L().oracle_diagmaxplus, init, (int(c),), table, want_col=True)


def min2plus_v(init, c: int = 1, table: bool = False) -> Result:
    """Vertical twin of min2plus ([L111], reading R15): f = min(L, UL) + c, column 0 = init.
    Returns score = min of the last column, last_col, table."""
    grid = _c(init, np.int32)
    H, W = grid.shape
    tab = np.empty((H, W), np.int32) if table else None
    last_col = np.empty(H, np.int32)
    score = _L().oracle_min2plus_v(_ptr(grid), H, W, int(c), _ptr(tab), W, _ptr(last_col))
    return Result(score=score, last_col=last_col, table=tab)


def antidiag_maxplus(init, c: int = 1, table: bool = False) -> Result:
    """mInverted-L twin of diagmaxplus ([L111], reading R15): f = max(init, UR) + c, row 0 and
    column W-1 = init.  Returns last_row and last_col = COLUMN 0 (where its chains end), table."""
    grid = _c(init, np.int32)
    H, W = grid.shape
    tab = np.empty((H, W), np.int32) if table else None
    last_row = np.empty(W, np.int32)
    first_col = np.empty(H, np.int32)
    _L().oracle_antidiag_maxplus(_ptr(grid), H, W, int(c), _ptr(tab), W, _ptr(last_row), _ptr(first_col))
    return Result(last_row=last_row, last_col=first_col, table=tab)


def traceback(func: str, a, b, table):
    """Traceback of a full oracle table (reading R14), plain Python loops: the DP cells
    (i, j), 1-based, visited from (m, n) while i >= 1 and j >= 1.  ``table[i-1][j-1] = D[i][j]``;
    row / column 0 are f's boundary.  LCS follows CLRS PRINT-LCS (match -> diagonal, else up when
    D[i-1][j] >= D[i][j-1]); Levenshtein takes a free diagonal on a match, else the first of
    substitution / deletion / insertion that reproduces D[i][j]; DTW the argmin of
    (UL, U, L), ties in that order, ending at (1, 1)."""
    m, n = len(a), len(b)
    inf = float("inf")

    def D(i, j):
        if i >= 1 and j >= 1:
            return table[i - 1][j - 1]
        if func == "levenshtein":
            return max(i, j)
        if func == "dtw":
            return 0.0 if i == 0 and j == 0 else inf
        return 0

    path = []
    i, j = m, n
    while i >= 1 and j >= 1:
        path.append((i, j))
        if func == "dtw":
            if i == 1 and j == 1:
                break
            d, u, l = D(i - 1, j - 1), D(i - 1, j), D(i, j - 1)
            if d <= u and d <= l:
                i, j = i - 1, j - 1
            elif u <= l:
                i -= 1
            else:
                j -= 1
        elif func == "lcs":
            if a[i - 1] == b[j - 1]:
                i, j = i - 1, j - 1
            elif D(i - 1, j) >= D(i, j - 1):
                i -= 1
            else:
                j -= 1
        else:
            here = D(i, j)
            if a[i - 1] == b[j - 1] and here == D(i - 1, j - 1):
                i, j = i - 1, j - 1
            elif here == D(i - 1, j - 1) + 1:
                i, j = i - 1, j - 1
            elif here == D(i - 1, j) + 1:
                i -= 1
            else:
                j -= 1
    return path


def lcs_string(a, b, path) -> bytes:
    """The common subsequence a LCS traceback path spells (matched diagonal moves)."""
    out = []
    for k, (i, j) in enumerate(path):
        nxt = path[k + 1] if k + 1 < len(path) else (i - 1, j - 1)
        if nxt == (i - 1, j - 1) and a[i - 1] == b[j - 1]:
            out.append(int(a[i - 1]))
    return bytes(reversed(out))
