"""ragen — seeded synthetic inputs shared by the oracle tests and the CUDA path.

INPUT GENERATION ONLY: this module holds none of the method's arithmetic
(no predicate evaluation, compaction, projection or aggregation).  It is the
one module both sides may use (task rule ③).  The generator itself lives in
``ragen_core.h``; ``libragen.so`` exposes a multithreaded host implementation
and a CUDA implementation of the same integer-only functions.

Recipes:

* ``int32_column`` — uniform over all 2^32 bit patterns ("random 32-bit
  integers", PAPER.md L493-494 / L990-993).
* ``lineitem`` — the seven Q1 columns with TPC-H
  §4.2.3 distributions restated in SURVEY.md C15, ``6_000_000 * SF`` rows.
* ``nested_thresholds`` — SURVEY C4: stage j of a chain keeps ``x < T_j`` with
  ``T_j = INT32_MIN + round(s**(j+1) * 2**32)`` so each SELECT keeps ~s of its
  own input ("two back-to-back SELECTs keep 25%").
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libragen.so")
_lib = None

ROWS_PER_SF = 6_000_000
PARTS_PER_SF = 200_000
INT32_MIN = -(2**31)
INT32_MAX = 2**31 - 1


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make` (or __graft_entry__.build())")
        L = ctypes.CDLL(_LIB_PATH)
        u64, i64, vp, i32, u32 = (ctypes.c_uint64, ctypes.c_int64, ctypes.c_void_p,
                                  ctypes.c_int, ctypes.c_uint32)
        L.ragen_int32_host.argtypes = [u64, u64, i64, vp, i32]
        L.ragen_int32_host.restype = None
        L.ragen_lineitem_host.argtypes = [u64, u32, u64, i64, vp, vp, vp, vp, vp, vp, vp, i32]
        L.ragen_lineitem_host.restype = None
        L.ragen_int32_dev.argtypes = [u64, u64, i64, vp, vp]
        L.ragen_int32_dev.restype = i32
        L.ragen_lineitem_dev.argtypes = [u64, u32, u64, i64, vp, vp, vp, vp, vp, vp, vp, vp]
        L.ragen_lineitem_dev.restype = i32
        _lib = L
    return _lib


def _nthreads() -> int:
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def rows_for_sf(sf: float) -> int:
    """exactly 6,000,000 x SF rows (not dbgen's 1-7 lines/order)."""
    return int(round(ROWS_PER_SF * sf))


def parts_for_sf(sf: float) -> int:
    return max(1, int(round(PARTS_PER_SF * sf)))


LINEITEM_COLUMNS = (
    ("shipdate", np.int32),
    ("returnflag", np.uint8),
    ("linestatus", np.uint8),
    ("quantity", np.int64),
    ("extendedprice", np.int64),
    ("discount", np.int64),
    ("tax", np.int64),
)


def int32_column(seed: int, n: int, row0: int = 0, out: np.ndarray | None = None) -> np.ndarray:
    if out is None:
        out = np.empty(n, dtype=np.int32)
    assert out.dtype == np.int32 and out.flags.c_contiguous and out.size >= n
    lib().ragen_int32_host(seed, row0, n, out.ctypes.data, _nthreads())
    return out


def lineitem(seed: int, n: int, n_parts: int, row0: int = 0, out: dict | None = None) -> dict:
    """Host lineitem columns for global rows [row0, row0+n) as numpy arrays."""
    if out is None:
        out = {name: np.empty(n, dtype=dt) for name, dt in LINEITEM_COLUMNS}
    ptrs = []
    for name, dt in LINEITEM_COLUMNS:
        a = out.get(name)
        if a is None:
            ptrs.append(None)
        else:
            assert a.dtype == dt and a.flags.c_contiguous and a.size >= n
            ptrs.append(a.ctypes.data)
    lib().ragen_lineitem_host(seed, n_parts, row0, n, *ptrs, _nthreads())
    return out


def int32_column_dev(seed: int, out, row0: int = 0, stream: int = 0) -> None:
    """Device generation into a CUDA int32 tensor ``out`` (same values as the host)."""
    rc = lib().ragen_int32_dev(seed, row0, out.numel(), out.data_ptr(), stream)
    if rc != 0:
        raise RuntimeError(f"ragen_int32_dev failed: cuda error {rc}")


def lineitem_dev(seed: int, n_parts: int, cols: dict, row0: int = 0, stream: int = 0) -> None:
    """Device generation into CUDA tensors ``cols[name]`` (same values as the host)."""
    n = cols["shipdate"].numel()
    ptrs = [cols[name].data_ptr() if name in cols else None for name, _ in LINEITEM_COLUMNS]
    rc = lib().ragen_lineitem_dev(seed, n_parts, row0, n, *ptrs, stream)
    if rc != 0:
        raise RuntimeError(f"ragen_lineitem_dev failed: cuda error {rc}")


def nested_thresholds(s: float, k: int) -> list[int]:
    """T_j = INT32_MIN + round(s^(j+1) * 2^32), j = 0..k-1 (LT predicates).

    s = 1 is not representable as an LT constant (C5); callers use GE INT32_MIN.
    """
    out = []
    for j in range(k):
        t = INT32_MIN + int(round((s ** (j + 1)) * 2**32))
        out.append(max(INT32_MIN, min(INT32_MAX, t)))
    return out
