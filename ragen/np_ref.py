"""Pure-numpy re-implementation of ragen_core.h — pins the C/CUDA generator.

Used only by tests (tests/test_ragen.py) to check that libragen.so produces
exactly the documented recipe; written independently from the C source using
uint64 wrap-around arithmetic.
"""
from __future__ import annotations

import numpy as np

M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_G = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def mix64(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = (z + _G).astype(np.uint64)
        z = ((z ^ (z >> np.uint64(30))) * _C1).astype(np.uint64)
        z = ((z ^ (z >> np.uint64(27))) * _C2).astype(np.uint64)
        return z ^ (z >> np.uint64(31))


def key(seed: int, stream: int) -> np.uint64:
    return mix64(np.array([(seed ^ (stream << 56)) & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64))[0]


def draw(k: np.uint64, idx: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        return mix64((idx.astype(np.uint64) + k).astype(np.uint64))


def uniform(h: np.ndarray, lo: int, span: int) -> np.ndarray:
    hi32 = (h >> np.uint64(32)).astype(np.uint64)
    return lo + ((hi32 * np.uint64(span)) >> np.uint64(32)).astype(np.int64)


def int32_column(seed: int, n: int, row0: int = 0) -> np.ndarray:
    idx = np.arange(row0, row0 + n, dtype=np.uint64)
    return (draw(key(seed, 0), idx) >> np.uint64(32)).astype(np.uint32).view(np.int32)


def lineitem(seed: int, n: int, n_parts: int, row0: int = 0) -> dict:
    idx = np.arange(row0, row0 + n, dtype=np.uint64)
    orderdate = uniform(draw(key(seed, 1), idx), 8035, 10440 - 8035 + 1)
    shipdate = orderdate + uniform(draw(key(seed, 2), idx), 1, 121)
    receipt = shipdate + uniform(draw(key(seed, 3), idx), 1, 30)
    coin = (draw(key(seed, 4), idx) >> np.uint64(63)).astype(np.int64)
    qty_units = uniform(draw(key(seed, 5), idx), 1, 50)
    disc = uniform(draw(key(seed, 6), idx), 0, 11)
    tax = uniform(draw(key(seed, 7), idx), 0, 9)
    pk = uniform(draw(key(seed, 8), idx), 1, max(1, n_parts))
    retail = 90000 + ((pk // 10) % 20001) + 100 * (pk % 1000)
    rf = np.where(receipt <= 9298, np.where(coin == 1, ord("R"), ord("A")), ord("N")).astype(np.uint8)
    ls = np.where(shipdate > 9298, ord("O"), ord("F")).astype(np.uint8)
    return {
        "shipdate": shipdate.astype(np.int32),
        "returnflag": rf,
        "linestatus": ls,
        "quantity": (qty_units * 100).astype(np.int64),
        "extendedprice": (qty_units * retail).astype(np.int64),
        "discount": disc.astype(np.int64),
        "tax": tax.astype(np.int64),
    }
