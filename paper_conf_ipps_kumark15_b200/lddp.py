"""Thin ctypes binding of liblddp.so (include/lddp.h) -- argument marshalling only.

Every step of the fill runs in the library's CUDA kernels; this module only converts torch
tensors / numpy arrays into the C structs and raises ``LddpError`` on a non-OK status.  The
functions keep the C names (``lddp_plan``, ``lddp_fill``, ...).  There is no CPU fallback:
importing this module without the built library raises ImportError.

Convenience layer: ``Plan`` wraps a plan handle and fills from torch CUDA tensors.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# LDDP_LIB_PATH: development A/B builds (make LIB=... BUILD=... EXTRA=...); default the in-tree build
LIB_PATH = os.environ.get("LDDP_LIB_PATH") or os.path.join(_HERE, "liblddp.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"liblddp.so not found at {LIB_PATH}: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
        "(or `make -C paper_conf_ipps_kumark15_b200`).  There is no CPU fallback.")
_lib = ctypes.CDLL(LIB_PATH)

# ---- enums (include/lddp.h) ---------------------------------------------------------------
LDDP_OK = 0
STATUS_NAMES = {0: "LDDP_OK", 1: "LDDP_ERR_INVALID_ARG", 2: "LDDP_ERR_SHAPE",
                3: "LDDP_ERR_CATEGORY_MISMATCH", 4: "LDDP_ERR_UNSUPPORTED",
                5: "LDDP_ERR_OUT_OF_MEMORY", 6: "LDDP_ERR_CUDA", 7: "LDDP_ERR_COMM",
                8: "LDDP_ERR_TIMEOUT", 9: "LDDP_ERR_INTERNAL"}
LDDP_ERR_INVALID_ARG, LDDP_ERR_SHAPE, LDDP_ERR_CATEGORY_MISMATCH, LDDP_ERR_UNSUPPORTED = 1, 2, 3, 4
LDDP_ERR_TIMEOUT = 8

CAT_PREV_ROW, CAT_ANTI_DIAGONAL, CAT_KNIGHT_MOVE, CAT_INVERTED_L, CAT_VERTICAL, CAT_MINVERTED_L = range(6)
CATEGORIES = {"prev_row": 0, "anti_diagonal": 1, "knight_move": 2, "inverted_l": 3, "vertical": 4,
              "minverted_l": 5}
PAT_HORIZONTAL, PAT_ANTI_DIAGONAL, PAT_KNIGHT_MOVE, PAT_INVERTED_L, PAT_VERTICAL, PAT_MINVERTED_L = range(6)
PATTERN_NAMES = {0: "Horizontal", 1: "Anti-diagonal", 2: "Knight-Move", 3: "Inverted-L",
                 4: "Vertical", 5: "mInverted-L"}
NB_L, NB_UL, NB_U, NB_UR = 1, 2, 4, 8
(F_LCS, F_DTW, F_FS_DITHER, F_MIN_PATH3, F_DIAG_MAXPLUS, F_MIN2_PLUS, F_LEVENSHTEIN, F_MIN2_PLUS_V,
 F_ANTIDIAG_MAXPLUS) = range(9)
FUNCS = {"lcs": 0, "dtw": 1, "fs": 2, "minpath3": 3, "diagmaxplus": 4, "min2plus": 5, "levenshtein": 6,
         "min2plus_v": 7, "antidiag_maxplus": 8}
OUT_SCORE, OUT_LAST_ROW, OUT_LAST_COL, OUT_TABLE = 1, 2, 4, 8
COMM_HANDLE_BYTES = 64


class lddp_desc(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64), ("category", ctypes.c_int32),
                ("func", ctypes.c_int32), ("outputs", ctypes.c_uint32), ("param_c", ctypes.c_int32),
                ("device", ctypes.c_int32), ("tile_rows", ctypes.c_int32),
                ("tile_warps", ctypes.c_int32), ("band_rows", ctypes.c_int32),
                ("grid_ctas", ctypes.c_int32), ("batch", ctypes.c_int32), ("reserved", ctypes.c_int32 * 2)]


class lddp_inputs(ctypes.Structure):
    _fields_ = [("a", ctypes.c_void_p), ("b", ctypes.c_void_p), ("grid", ctypes.c_void_p),
                ("grid_pitch", ctypes.c_int64)]


class lddp_outputs(ctypes.Structure):
    _fields_ = [("score", ctypes.c_void_p), ("last_row", ctypes.c_void_p),
                ("last_col", ctypes.c_void_p), ("table", ctypes.c_void_p),
                ("table_pitch", ctypes.c_int64)]


_P = ctypes.c_void_p
_SIGS = {
    "lddp_abi_version": (ctypes.c_int32, []),
    "lddp_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "lddp_last_error_message": (ctypes.c_char_p, []),
    "lddp_func_mask": (ctypes.c_int, [ctypes.c_int32, ctypes.POINTER(ctypes.c_uint32)]),
    "lddp_classify": (ctypes.c_int, [ctypes.c_uint32, ctypes.POINTER(ctypes.c_int32)]),
    "lddp_category_covers": (ctypes.c_int, [ctypes.c_int32, ctypes.c_uint32, ctypes.POINTER(ctypes.c_int32)]),
    "lddp_plan": (ctypes.c_int, [ctypes.POINTER(lddp_desc), ctypes.POINTER(_P)]),
    "lddp_plan_destroy": (ctypes.c_int, [_P]),
    "lddp_plan_workspace_size": (ctypes.c_int, [_P, ctypes.POINTER(ctypes.c_size_t)]),
    "lddp_plan_describe": (ctypes.c_int, [_P, ctypes.c_char_p, ctypes.c_size_t]),
    "lddp_workspace_init": (ctypes.c_int, [_P, _P, _P]),
    "lddp_fill": (ctypes.c_int, [_P, ctypes.POINTER(lddp_inputs), ctypes.POINTER(lddp_outputs), _P, _P]),
    "lddp_fill_host": (ctypes.c_int, [_P, ctypes.POINTER(lddp_inputs), ctypes.POINTER(lddp_outputs), _P]),
    "lddp_status_check": (ctypes.c_int, [_P, _P, _P]),
    "lddp_comm_create": (ctypes.c_int, [_P, ctypes.c_int32, ctypes.c_int32, ctypes.POINTER(_P)]),
    "lddp_comm_handle": (ctypes.c_int, [_P, ctypes.c_char_p]),
    "lddp_comm_connect": (ctypes.c_int, [_P, ctypes.c_char_p, ctypes.c_char_p]),
    "lddp_comm_connect_local": (ctypes.c_int, [_P, _P, _P]),
    "lddp_plan_partition": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                           ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]),
    "lddp_multi_partition": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                            ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]),
    "lddp_comm_destroy": (ctypes.c_int, [_P]),
    "lddp_fill_multi": (ctypes.c_int, [_P, ctypes.POINTER(lddp_inputs), ctypes.POINTER(lddp_outputs), _P, _P, _P]),
    "lddp_traceback": (ctypes.c_int, [_P, ctypes.POINTER(lddp_inputs), _P, ctypes.c_int64, _P, _P, _P, _P]),
}
for _name, (_res, _args) in _SIGS.items():
    _fn = getattr(_lib, _name)
    _fn.restype = _res
    _fn.argtypes = _args

EXPORTED = tuple(_SIGS)


class LddpError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        msg = _lib.lddp_last_error_message().decode(errors="replace")
        super().__init__(f"{where}: {STATUS_NAMES.get(status, status)}: {msg}")


def _check(st, where):
    if st != LDDP_OK:
        raise LddpError(st, where)


# ---- same-name wrappers ---------------------------------------------------------------------
def lddp_abi_version() -> int:
    return _lib.lddp_abi_version()


def lddp_func_mask(func: int) -> int:
    m = ctypes.c_uint32()
    _check(_lib.lddp_func_mask(func, ctypes.byref(m)), "lddp_func_mask")
    return m.value


def lddp_classify(mask: int) -> int:
    p = ctypes.c_int32()
    _check(_lib.lddp_classify(mask, ctypes.byref(p)), "lddp_classify")
    return p.value


def lddp_category_covers(category: int, mask: int) -> bool:
    c = ctypes.c_int32()
    _check(_lib.lddp_category_covers(category, mask, ctypes.byref(c)), "lddp_category_covers")
    return bool(c.value)


def lddp_plan(desc: lddp_desc):
    h = _P()
    _check(_lib.lddp_plan(ctypes.byref(desc), ctypes.byref(h)), "lddp_plan")
    return h


def lddp_plan_destroy(plan) -> None:
    _check(_lib.lddp_plan_destroy(plan), "lddp_plan_destroy")


def lddp_plan_workspace_size(plan) -> int:
    n = ctypes.c_size_t()
    _check(_lib.lddp_plan_workspace_size(plan, ctypes.byref(n)), "lddp_plan_workspace_size")
    return n.value


def lddp_plan_describe(plan) -> str:
    buf = ctypes.create_string_buffer(1024)
    _check(_lib.lddp_plan_describe(plan, buf, len(buf)), "lddp_plan_describe")
    return buf.value.decode()


def lddp_workspace_init(plan, ws_ptr: int, stream: int = 0) -> None:
    _check(_lib.lddp_workspace_init(plan, ws_ptr, stream), "lddp_workspace_init")


def lddp_fill(plan, inputs: lddp_inputs, outputs: lddp_outputs, ws_ptr, stream: int = 0) -> None:
    _check(_lib.lddp_fill(plan, ctypes.byref(inputs), ctypes.byref(outputs), ws_ptr, stream), "lddp_fill")


def lddp_fill_host(plan, inputs: lddp_inputs, outputs: lddp_outputs, stream: int = 0) -> None:
    _check(_lib.lddp_fill_host(plan, ctypes.byref(inputs), ctypes.byref(outputs), stream), "lddp_fill_host")


def lddp_status_check(plan, ws_ptr=None, stream: int = 0) -> None:
    _check(_lib.lddp_status_check(plan, ws_ptr, stream), "lddp_status_check")


def lddp_comm_create(plan, nranks: int, rank: int):
    h = _P()
    _check(_lib.lddp_comm_create(plan, nranks, rank, ctypes.byref(h)), "lddp_comm_create")
    return h


def lddp_comm_handle(comm) -> bytes:
    buf = ctypes.create_string_buffer(COMM_HANDLE_BYTES)
    _check(_lib.lddp_comm_handle(comm, buf), "lddp_comm_handle")
    return buf.raw


def lddp_comm_connect(comm, next_handle, prev_handle=None) -> None:
    """next_handle: rank g+1's window handle (None on the last rank); prev_handle: rank g-1's
    (None on rank 0)."""
    _check(_lib.lddp_comm_connect(comm, next_handle, prev_handle), "lddp_comm_connect")


def lddp_comm_connect_local(comm, next_comm, prev_comm=None) -> None:
    _check(_lib.lddp_comm_connect_local(comm, next_comm, prev_comm), "lddp_comm_connect_local")


def lddp_multi_partition(cols: int, nranks: int, rank: int):
    """Columns [c0, c1) rank `rank` of `nranks` owns (host only, no GPU needed)."""
    c0, c1 = ctypes.c_int64(), ctypes.c_int64()
    _check(_lib.lddp_multi_partition(cols, nranks, rank, ctypes.byref(c0), ctypes.byref(c1)),
           "lddp_multi_partition")
    return c0.value, c1.value


def lddp_plan_partition(plan, nranks: int, rank: int):
    lo, hi = ctypes.c_int64(), ctypes.c_int64()
    _check(_lib.lddp_plan_partition(plan, nranks, rank, ctypes.byref(lo), ctypes.byref(hi)),
           "lddp_plan_partition")
    return lo.value, hi.value


def lddp_comm_destroy(comm) -> None:
    _check(_lib.lddp_comm_destroy(comm), "lddp_comm_destroy")


def lddp_fill_multi(plan, inputs, outputs, ws_ptr, comm, stream: int = 0) -> None:
    _check(_lib.lddp_fill_multi(plan, ctypes.byref(inputs), ctypes.byref(outputs), ws_ptr, comm, stream),
           "lddp_fill_multi")


# ---- torch convenience layer ----------------------------------------------------------------
def _ptr(t):
    return None if t is None else t.data_ptr()


def _stream_handle(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


class Plan:
    """A plan plus its workspace (torch uint8 tensor on the plan's device)."""

    def __init__(self, func, category, rows, cols, outputs, param_c=1, device=0, tile_rows=0,
                 grid_ctas=0, band_rows=0, batch=0):
        import torch
        self.func = FUNCS[func] if isinstance(func, str) else int(func)
        self.category = CATEGORIES[category] if isinstance(category, str) else int(category)
        self.rows, self.cols, self.outputs = int(rows), int(cols), int(outputs)
        self.device = int(device)
        self.desc = lddp_desc(rows=self.rows, cols=self.cols, category=self.category, func=self.func,
                              outputs=self.outputs, param_c=int(param_c), device=self.device,
                              tile_rows=int(tile_rows), tile_warps=0, band_rows=int(band_rows),
                              grid_ctas=int(grid_ctas), batch=int(batch))
        self.handle = lddp_plan(self.desc)
        self.ws_bytes = lddp_plan_workspace_size(self.handle)
        self.ws = torch.zeros(max(self.ws_bytes, 64), dtype=torch.uint8, device=f"cuda:{self.device}")
        self.info = lddp_plan_describe(self.handle)

    def __del__(self):
        h = getattr(self, "handle", None)
        if h:
            try:
                lddp_plan_destroy(h)
            except Exception:
                pass
            self.handle = None

    @staticmethod
    def io(a=None, b=None, grid=None, score=None, last_row=None, last_col=None, table=None):
        inp = lddp_inputs(a=_ptr(a), b=_ptr(b), grid=_ptr(grid),
                          grid_pitch=0 if grid is None else grid.stride(0))
        out = lddp_outputs(score=_ptr(score), last_row=_ptr(last_row), last_col=_ptr(last_col),
                           table=_ptr(table), table_pitch=0 if table is None else table.stride(0))
        return inp, out

    def fill(self, stream=None, **tensors):
        inp, out = self.io(**tensors)
        lddp_fill(self.handle, inp, out, self.ws.data_ptr(), _stream_handle(stream))

    def check(self, stream=None):
        lddp_status_check(self.handle, self.ws.data_ptr(), _stream_handle(stream))

    def traceback(self, a, b, table, stream=None):
        """Traceback of this plan's TABLE output (LCS / Levenshtein / DTW) on the device: returns
        the visited DP cells (i, j), 1-based, from (m, n) backwards, as two int32 device tensors."""
        import torch

        cap = max(self.rows + self.cols, 1)
        pi = torch.empty(cap, dtype=torch.int32, device=table.device)
        pj = torch.empty(cap, dtype=torch.int32, device=table.device)
        ln = torch.zeros(1, dtype=torch.int64, device=table.device)
        inp = lddp_inputs(a=_ptr(a), b=_ptr(b), grid=None, grid_pitch=0)
        _check(_lib.lddp_traceback(self.handle, ctypes.byref(inp), _ptr(table), table.stride(0), _ptr(pi), _ptr(pj),
                                   _ptr(ln), _stream_handle(stream)), "lddp_traceback")
        k = int(ln.item())
        return pi[:k], pj[:k]
