"""CPU oracle (ctypes wrapper around oracle/liboracle.so, built from oracle.c).

TEST INFRASTRUCTURE ONLY.  Only tests/, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with the CUDA path and never imports it.

Predicates are given as ``(op_name, value)`` pairs with op names
``"lt" "le" "gt" "ge" "eq" "ne"``; this module maps them to the
oracle's own op codes.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

OPS = {"lt": 0, "le": 1, "gt": 2, "ge": 3, "eq": 4, "ne": 5}


class _Pred(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("value", ctypes.c_int32)]


class Q1Row(ctypes.Structure):
    _fields_ = [
        ("returnflag", ctypes.c_uint8),
        ("linestatus", ctypes.c_uint8),
        ("_pad", ctypes.c_uint8 * 6),
        ("count_order", ctypes.c_int64),
        ("sum_qty_lo", ctypes.c_uint64),
        ("sum_qty_hi", ctypes.c_int64),
        ("sum_base_price_lo", ctypes.c_uint64),
        ("sum_base_price_hi", ctypes.c_int64),
        ("sum_disc_price_lo", ctypes.c_uint64),
        ("sum_disc_price_hi", ctypes.c_int64),
        ("sum_charge_lo", ctypes.c_uint64),
        ("sum_charge_hi", ctypes.c_int64),
        ("sum_disc_lo", ctypes.c_uint64),
        ("sum_disc_hi", ctypes.c_int64),
        ("avg_qty", ctypes.c_double),
        ("avg_price", ctypes.c_double),
        ("avg_disc", ctypes.c_double),
    ]


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make`")
        L = ctypes.CDLL(_LIB_PATH)
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        for name in ("oracle_select", "oracle_select_unfused"):
            f = getattr(L, name)
            f.argtypes = [vp, i64, vp, i32, vp]
            f.restype = i64
        L.oracle_select_chunked.argtypes = [vp, i64, vp, i32, i64, vp]
        L.oracle_select_chunked.restype = i64
        L.oracle_select_multi.argtypes = [vp, i64, vp, vp, vp, i32, vp, vp]
        L.oracle_select_multi.restype = i32
        L.oracle_select_rows.argtypes = [vp, i64, vp, i32, i32, vp, vp, vp, vp]
        L.oracle_select_rows.restype = i64
        L.oracle_q1.argtypes = [vp, vp, vp, vp, vp, vp, vp, i64, ctypes.c_int32, vp, vp]
        L.oracle_q1.restype = i32
        L.oracle_q1_row_size.restype = i32
        assert L.oracle_q1_row_size() == ctypes.sizeof(Q1Row)
        _lib = L
    return _lib


def _preds(preds):
    arr = (_Pred * max(1, len(preds)))()
    for i, (op, v) in enumerate(preds):
        arr[i].op = OPS[op] if isinstance(op, str) else int(op)
        arr[i].value = int(v)
    return arr


def _as_i32(x) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.int32)
    return x


def select(x, preds, fused: bool = True) -> np.ndarray:
    """Order-preserving SELECT of x by the conjunction of ``preds``."""
    x = _as_i32(x)
    P = _preds(preds)
    out = np.empty(max(1, x.size), dtype=np.int32)
    f = lib().oracle_select if fused else lib().oracle_select_unfused
    m = f(x.ctypes.data, x.size, ctypes.addressof(P), len(preds), out.ctypes.data)
    if m < 0:
        raise ValueError(f"oracle_select failed ({m})")
    return out[:m].copy()


def select_count(x, preds) -> int:
    x = _as_i32(x)
    P = _preds(preds)
    m = lib().oracle_select(x.ctypes.data, x.size, ctypes.addressof(P), len(preds), None)
    if m < 0:
        raise ValueError(f"oracle_select failed ({m})")
    return int(m)


def select_chunked(x, preds, chunk: int) -> np.ndarray:
    x = _as_i32(x)
    P = _preds(preds)
    out = np.empty(max(1, x.size), dtype=np.int32)
    m = lib().oracle_select_chunked(x.ctypes.data, x.size, ctypes.addressof(P),
                                    len(preds), chunk, out.ctypes.data)
    if m < 0:
        raise ValueError(f"oracle_select_chunked failed ({m})")
    return out[:m].copy()


def select_multi(x, chains):
    """Several SELECTs on the same input (Fig 2(c)): one order-preserving
    output per predicate chain in ``chains``."""
    x = _as_i32(x)
    flat = [p for c in chains for p in c]
    P = _preds(flat)
    M = len(chains)
    off = (ctypes.c_int32 * max(1, M))(*[sum(len(c) for c in chains[:o]) for o in range(M)])
    ks = (ctypes.c_int32 * max(1, M))(*[len(c) for c in chains])
    outs = [np.empty(max(1, x.size), dtype=np.int32) for _ in range(M)]
    op = (ctypes.c_void_p * max(1, M))(*[o.ctypes.data for o in outs])
    counts = np.zeros(max(1, M), dtype=np.int64)
    rc = lib().oracle_select_multi(x.ctypes.data, x.size, ctypes.addressof(P), ctypes.addressof(off),
                                   ctypes.addressof(ks), M, ctypes.addressof(op), counts.ctypes.data)
    if rc < 0:
        raise ValueError(f"oracle_select_multi failed ({rc})")
    return [o[:c].copy() for o, c in zip(outs, counts[:M])]


def select_rows(key, preds, payloads=()):
    """SELECT over a multi-column relation (Table I): the predicate chain on
    the int32 key column; returns ``(rowids int64, [payload[rowids] ...])``
    with rows in input order.  Payload columns are 4- or 8-byte arrays."""
    key = _as_i32(key)
    P = _preds(preds)
    cols = [np.ascontiguousarray(c) for c in payloads]
    for c in cols:
        if c.size != key.size or c.dtype.itemsize not in (4, 8):
            raise ValueError("payload columns must match the key length and be 4- or 8-byte")
    m = len(cols)
    rowids = np.empty(max(1, key.size), dtype=np.int64)
    outs = [np.empty(max(1, key.size), dtype=c.dtype) for c in cols]
    cp = (ctypes.c_void_p * max(1, m))(*[c.ctypes.data for c in cols])
    eb = (ctypes.c_int32 * max(1, m))(*[c.dtype.itemsize for c in cols])
    op = (ctypes.c_void_p * max(1, m))(*[o.ctypes.data for o in outs])
    cnt = lib().oracle_select_rows(key.ctypes.data, key.size, ctypes.addressof(P), len(preds), m,
                                   ctypes.addressof(cp), ctypes.addressof(eb), rowids.ctypes.data,
                                   ctypes.addressof(op))
    if cnt < 0:
        raise ValueError(f"oracle_select_rows failed ({cnt})")
    return rowids[:cnt].copy(), [o[:cnt].copy() for o in outs]


def _i128(lo: int, hi: int) -> int:
    return (int(hi) << 64) | int(lo)


def q1(cols: dict, cutoff: int = 10471):
    """TPC-H Q1 over lineitem columns.  Returns (rows, status).

    Each row is a dict with exact Python-int sums (scaled integers: qty/price/
    disc x100, disc_price x1e4, charge x1e6) and the three AVG doubles.
    """
    n = int(cols["shipdate"].size)
    arrs = [
        np.ascontiguousarray(cols["shipdate"], dtype=np.int32),
        np.ascontiguousarray(cols["returnflag"], dtype=np.uint8),
        np.ascontiguousarray(cols["linestatus"], dtype=np.uint8),
        np.ascontiguousarray(cols["quantity"], dtype=np.int64),
        np.ascontiguousarray(cols["extendedprice"], dtype=np.int64),
        np.ascontiguousarray(cols["discount"], dtype=np.int64),
        np.ascontiguousarray(cols["tax"], dtype=np.int64),
    ]
    rows = (Q1Row * 65536)()
    status = ctypes.c_uint32(0)
    m = lib().oracle_q1(*[a.ctypes.data for a in arrs], n, int(cutoff), ctypes.addressof(rows),
                        ctypes.addressof(status))
    if m < 0:
        raise MemoryError("oracle_q1 failed")
    out = []
    for r in rows[:m]:
        out.append({
            "returnflag": chr(r.returnflag) if r.returnflag < 128 else r.returnflag,
            "linestatus": chr(r.linestatus) if r.linestatus < 128 else r.linestatus,
            "rf_byte": r.returnflag,
            "ls_byte": r.linestatus,
            "count_order": r.count_order,
            "sum_qty": _i128(r.sum_qty_lo, r.sum_qty_hi),
            "sum_base_price": _i128(r.sum_base_price_lo, r.sum_base_price_hi),
            "sum_disc_price": _i128(r.sum_disc_price_lo, r.sum_disc_price_hi),
            "sum_charge": _i128(r.sum_charge_lo, r.sum_charge_hi),
            "sum_disc": _i128(r.sum_disc_lo, r.sum_disc_hi),
            "avg_qty": r.avg_qty,
            "avg_price": r.avg_price,
            "avg_disc": r.avg_disc,
        })
    return out, int(status.value)
