"""ctypes binding of libra.so — argument marshalling only.

Every function named ``ra_*`` mirrors the C entry point of the same name in
``include/ra.h`` (same arguments, same order; pointers as ints, streams as
``cudaStream_t`` ints) and raises ``RAError`` on a negative return code.
No step of the hot path runs here: all of it runs in libra.so's kernels.
There is no fallback — importing this module fails if libra.so is missing.
"""
from __future__ import annotations

import ctypes
import os
import re

_HERE = os.path.dirname(os.path.abspath(__file__))
# RA_LIB_PATH: load a diagnostics build of libra.so (scripts/; e.g. compile-time
# variants or the watchdog build).  Tests, smoke() and bench.py never set it.
LIB_PATH = os.environ.get("RA_LIB_PATH") or os.path.join(_HERE, "libra.so")
HEADER_PATH = os.path.join(os.path.dirname(_HERE), "include", "ra.h")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `make` (or __graft_entry__.build()); "
                      "there is no non-CUDA fallback")

_lib = ctypes.CDLL(LIB_PATH)

RA_OK = 0
RA_E_INVAL = -1
RA_E_CAPACITY = -2
RA_E_DOMAIN = -3
RA_E_NOT_PINNED = -4
RA_E_CUDA = -5
RA_E_WORKSPACE = -6
RA_MAX_PREDS = 8
RA_MAX_PAYLOAD = 4
RA_MAX_OUTPUTS = 4
RA_MAX_RANKS = 65536
RA_Q1_GROUPS = 6
RA_LT, RA_LE, RA_GT, RA_GE, RA_EQ, RA_NE = range(6)
OPS = {"lt": RA_LT, "le": RA_LE, "gt": RA_GT, "ge": RA_GE, "eq": RA_EQ, "ne": RA_NE}

_ERRNAMES = {RA_E_INVAL: "RA_E_INVAL", RA_E_CAPACITY: "RA_E_CAPACITY", RA_E_DOMAIN: "RA_E_DOMAIN",
             RA_E_NOT_PINNED: "RA_E_NOT_PINNED", RA_E_CUDA: "RA_E_CUDA", RA_E_WORKSPACE: "RA_E_WORKSPACE"}


class RAError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_ERRNAMES.get(code, code)}: {msg}")
        self.code = code


class ra_pred(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("value", ctypes.c_int32)]


class ra_payload(ctypes.Structure):
    _fields_ = [("col", ctypes.c_void_p), ("out", ctypes.c_void_p), ("elem_bytes", ctypes.c_int32),
                ("_pad", ctypes.c_int32)]


class ra_lineitem(ctypes.Structure):
    _fields_ = [(name, ctypes.c_void_p) for name in (
        "shipdate", "returnflag", "linestatus", "quantity", "extendedprice", "discount", "tax")]


class ra_lineitem_narrow(ctypes.Structure):
    _fields_ = [(name, ctypes.c_void_p) for name in (
        "shipdate", "group", "quantity", "discount", "tax", "extendedprice")]


class ra_lineitem_narrow_out(ctypes.Structure):
    _fields_ = [(name, ctypes.c_void_p) for name in (
        "shipdate", "group", "quantity", "discount", "tax", "extendedprice")]


class ra_q1_group(ctypes.Structure):
    _fields_ = [
        ("count", ctypes.c_int64),
        ("sum_qty", ctypes.c_int64),
        ("sum_base_price", ctypes.c_int64),
        ("sum_disc", ctypes.c_int64),
        ("sum_disc_price_lo", ctypes.c_uint64),
        ("sum_disc_price_hi", ctypes.c_int64),
        ("sum_charge_lo", ctypes.c_uint64),
        ("sum_charge_hi", ctypes.c_int64),
    ]


class ra_q1_partial(ctypes.Structure):
    _fields_ = [
        ("status", ctypes.c_uint32),
        ("n_groups", ctypes.c_uint32),
        ("rows", ctypes.c_uint64),
        ("group", ra_q1_group * RA_Q1_GROUPS),
    ]


class ra_q1_row(ctypes.Structure):
    _fields_ = [
        ("returnflag", ctypes.c_uint8),
        ("linestatus", ctypes.c_uint8),
        ("_pad", ctypes.c_uint8 * 6),
        ("count_order", ctypes.c_int64),
        ("sum_qty", ctypes.c_int64),
        ("sum_base_price", ctypes.c_int64),
        ("sum_disc", ctypes.c_int64),
        ("sum_disc_price_lo", ctypes.c_uint64),
        ("sum_disc_price_hi", ctypes.c_int64),
        ("sum_charge_lo", ctypes.c_uint64),
        ("sum_charge_hi", ctypes.c_int64),
        ("avg_qty", ctypes.c_double),
        ("avg_price", ctypes.c_double),
        ("avg_disc", ctypes.c_double),
    ]


_vp, _i64, _i32, _sz = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_size_t
_SIGS = {
    "ra_last_error": ([], ctypes.c_char_p),
    "ra_version": ([], _i32),
    "ra_kernel_launches": ([], ctypes.c_uint64),
    "ra_workspace_init": ([_vp, _sz, _vp], _i32),
    "ra_select_workspace_bytes": ([_i64, _i32, _i32], _sz),
    "ra_select": ([_vp, _i64, ra_pred, _vp, _i64, _vp, _vp, _sz, _vp], _i32),
    "ra_select_chain": ([_vp, _i64, _vp, _i32, _i32, _vp, _i64, _vp, _vp, _sz, _vp], _i32),
    "ra_select_multi": ([_vp, _i64, _vp, _vp, _i32, _vp, _vp, _vp, _vp, _sz, _vp], _i32),
    "ra_select_offsets": ([_vp, _i32, _vp, _vp, _vp], _i32),
    "ra_select_rows_workspace_bytes": ([_i64, _i32], _sz),
    "ra_select_multi_workspace_bytes": ([_i64], _sz),
    "ra_select_rows": ([_vp, _i64, _vp, _i32, _vp, _vp, _i32, _i64, _vp, _vp, _sz, _vp], _i32),
    "ra_q1_workspace_bytes": ([_i64], _sz),
    "ra_q1": ([_vp, _i64, ctypes.c_int32, _vp, _vp, _sz, _vp], _i32),
    "ra_q1_finalize": ([_vp, _i32, _vp, _vp], _i32),
    "ra_fission_workspace_bytes": ([_i64, _i32, _i32, _i32], _sz),
    "ra_fission_run": ([_vp, _i64, _vp, _i32, _i32, _i64, _vp, _i32, _vp, _i64, _vp, _vp, _vp, _sz], _i32),
    "ra_q1_fission_workspace_bytes": ([_i64, _i32], _sz),
    "ra_q1_fission_run": ([_vp, _i64, ctypes.c_int32, _i64, _vp, _i32, _vp, _vp, _sz], _i32),
    "ra_q1_encode": ([_vp, _i64, _vp, _vp, _vp], _i32),
    "ra_q1_narrow": ([_vp, _i64, ctypes.c_int32, _vp, _vp, _sz, _vp], _i32),
    "ra_q1_narrow_fission_workspace_bytes": ([_i64, _i32], _sz),
    "ra_q1_narrow_fission_run": ([_vp, _i64, ctypes.c_int32, _i64, _vp, _i32, _vp, _vp, _sz], _i32),
}
for _name, (_args, _res) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res


def exported_symbols_from_header(path: str = HEADER_PATH) -> list[str]:
    """Function names declared in include/ra.h (used by the ABI test)."""
    with open(path) as f:
        src = f.read()
    return sorted(set(re.findall(r"^\s*(?:const\s+)?[\w\s\*]+?\b(ra_\w+)\s*\(", src, re.M)))


def _check(rc: int) -> int:
    if rc < 0:
        raise RAError(rc, ra_last_error())
    return rc


def ra_last_error() -> str:
    return (_lib.ra_last_error() or b"").decode()


def ra_version() -> int:
    return _lib.ra_version()


def ra_kernel_launches() -> int:
    return int(_lib.ra_kernel_launches())


def ra_workspace_init(d_ws: int, ws_bytes: int, stream: int) -> None:
    _check(_lib.ra_workspace_init(d_ws, ws_bytes, stream))


def ra_select_workspace_bytes(n: int, k: int, fused: int) -> int:
    return int(_lib.ra_select_workspace_bytes(n, k, fused))


def ra_select(d_in: int, n: int, pred: ra_pred, d_out: int, out_cap: int, d_count: int, d_ws: int,
              ws_bytes: int, stream: int) -> None:
    _check(_lib.ra_select(d_in, n, pred, d_out, out_cap, d_count, d_ws, ws_bytes, stream))


def ra_select_chain(d_in: int, n: int, h_preds, k: int, fused: int, d_out: int, out_cap: int,
                    d_count: int, d_ws: int, ws_bytes: int, stream: int) -> None:
    _check(_lib.ra_select_chain(d_in, n, h_preds, k, fused, d_out, out_cap, d_count, d_ws, ws_bytes,
                                stream))


def ra_select_offsets(d_counts: int, n_ranks: int, d_offsets: int, d_total: int, stream: int) -> None:
    _check(_lib.ra_select_offsets(d_counts, n_ranks, d_offsets, d_total, stream))


def ra_select_multi(d_in: int, n: int, h_chains, ks, M: int, d_outs, out_caps, d_counts, d_ws: int,
                    ws_bytes: int, stream: int) -> None:
    _check(_lib.ra_select_multi(d_in, n, h_chains, ks, M, d_outs, out_caps, d_counts, d_ws, ws_bytes, stream))


def ra_select_multi_workspace_bytes(n: int) -> int:
    return int(_lib.ra_select_multi_workspace_bytes(n))


def ra_select_rows_workspace_bytes(n: int, k: int) -> int:
    return int(_lib.ra_select_rows_workspace_bytes(n, k))


def ra_select_rows(d_key: int, n: int, h_preds, k: int, d_rowids: int, h_payloads, m: int, out_cap: int,
                   d_count: int, d_ws: int, ws_bytes: int, stream: int) -> None:
    _check(_lib.ra_select_rows(d_key, n, h_preds, k, d_rowids, h_payloads, m, out_cap, d_count, d_ws, ws_bytes,
                               stream))


def ra_q1_workspace_bytes(n: int) -> int:
    return int(_lib.ra_q1_workspace_bytes(n))


def ra_q1(h_cols: ra_lineitem, n: int, cutoff: int, d_partial: int, d_ws: int, ws_bytes: int,
          stream: int) -> None:
    _check(_lib.ra_q1(ctypes.byref(h_cols), n, cutoff, d_partial, d_ws, ws_bytes, stream))


def ra_q1_finalize(h_partials, n_partials: int, h_rows, n_rows) -> int:
    """Returns the raw code (RA_OK or RA_E_DOMAIN) — rows are filled either way."""
    rc = _lib.ra_q1_finalize(h_partials, n_partials, h_rows, n_rows)
    if rc < 0 and rc != RA_E_DOMAIN:
        raise RAError(rc, ra_last_error())
    return rc


def ra_fission_workspace_bytes(chunk_rows: int, n_streams: int, k: int, fused: int) -> int:
    return int(_lib.ra_fission_workspace_bytes(chunk_rows, n_streams, k, fused))


def ra_fission_run(h_in: int, n: int, h_preds, k: int, fused: int, chunk_rows: int, streams,
                   n_streams: int, h_out: int, out_cap: int, h_count, h_chunk_counts: int, d_ws: int,
                   ws_bytes: int) -> int:
    """Returns RA_OK or RA_E_CAPACITY (count still valid); raises on other errors."""
    rc = _lib.ra_fission_run(h_in, n, h_preds, k, fused, chunk_rows, streams, n_streams, h_out, out_cap,
                             h_count, h_chunk_counts, d_ws, ws_bytes)
    if rc < 0 and rc != RA_E_CAPACITY:
        raise RAError(rc, ra_last_error())
    return rc


def ra_q1_fission_workspace_bytes(chunk_rows: int, n_streams: int) -> int:
    return int(_lib.ra_q1_fission_workspace_bytes(chunk_rows, n_streams))


def ra_q1_fission_run(h_cols: ra_lineitem, n: int, cutoff: int, chunk_rows: int, streams, n_streams: int,
                      h_partial, d_ws: int, ws_bytes: int) -> None:
    _check(_lib.ra_q1_fission_run(ctypes.byref(h_cols), n, cutoff, chunk_rows, streams, n_streams,
                                  ctypes.byref(h_partial), d_ws, ws_bytes))


def ra_q1_encode(h_cols: ra_lineitem, n: int, h_out: ra_lineitem_narrow_out, d_status: int, stream: int) -> None:
    _check(_lib.ra_q1_encode(ctypes.byref(h_cols), n, ctypes.byref(h_out), d_status, stream))


def ra_q1_narrow(h_cols: ra_lineitem_narrow, n: int, cutoff: int, d_partial: int, d_ws: int, ws_bytes: int,
                 stream: int) -> None:
    _check(_lib.ra_q1_narrow(ctypes.byref(h_cols), n, cutoff, d_partial, d_ws, ws_bytes, stream))


def ra_q1_narrow_fission_workspace_bytes(chunk_rows: int, n_streams: int) -> int:
    return int(_lib.ra_q1_narrow_fission_workspace_bytes(chunk_rows, n_streams))


def ra_q1_narrow_fission_run(h_cols: ra_lineitem_narrow, n: int, cutoff: int, chunk_rows: int, streams,
                             n_streams: int, h_partial, d_ws: int, ws_bytes: int) -> None:
    _check(_lib.ra_q1_narrow_fission_run(ctypes.byref(h_cols), n, cutoff, chunk_rows, streams, n_streams,
                                         ctypes.byref(h_partial), d_ws, ws_bytes))


def make_preds(preds):
    """[(op_name_or_code, value), ...] -> ctypes ra_pred array (kept alive by the caller)."""
    arr = (ra_pred * max(1, len(preds)))()
    for i, (op, v) in enumerate(preds):
        arr[i].op = OPS[op] if isinstance(op, str) else int(op)
        arr[i].value = int(v)
    return arr
