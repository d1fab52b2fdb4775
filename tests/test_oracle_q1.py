"""Pins for the oracle's TPC-H Q1.

Ties oracle/oracle.c's Q1 to: a hand-computed fixture (tests/golden/
q1_worked_example.txt), pure-Python exact-integer brute force, pyarrow
decimal128 group_by (exact decimal arithmetic, a library routine), sqlite3
(exact int64 SUM, raises on overflow), Fraction-rounded AVG, and invariants
(count sums, cutoff extremes, partition additivity).
"""
import sqlite3
from fractions import Fraction

import numpy as np
import pytest

import oracle
import ragen
from golden_io import q1_worked_example, rows_to_columns

CUTOFF = 10471  # 1998-09-02 = 1998-12-01 - 90 days
SUMS = ("count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc")


def brute_q1(cols, cutoff):
    """Pure-Python Q1 with exact ints (tiny inputs only)."""
    acc = {}
    n = cols["shipdate"].size
    for i in range(n):
        if int(cols["shipdate"][i]) > cutoff:
            continue
        g = (int(cols["returnflag"][i]), int(cols["linestatus"][i]))
        q, p, d, t = (int(cols[c][i]) for c in ("quantity", "extendedprice", "discount", "tax"))
        a = acc.setdefault(g, [0, 0, 0, 0, 0, 0])
        a[0] += 1
        a[1] += q
        a[2] += p
        a[3] += p * (100 - d)
        a[4] += p * (100 - d) * (100 + t)
        a[5] += d
    return {g: a for g, a in sorted(acc.items())}


def test_worked_example():
    cutoff, rows, expect = q1_worked_example()
    got, status = oracle.q1(rows_to_columns(rows), cutoff)
    assert status == 0
    assert len(got) == len(expect)
    for g, e in zip(got, expect):
        for k, v in e.items():
            assert g[k] == v, (k, g[k], v)


def _random_cols(rng, n, bytes_domain=True):
    cols = ragen.lineitem(int(rng.integers(1 << 30)), n, 2000)
    if not bytes_domain:
        cols["returnflag"][rng.integers(0, n, 3)] = rng.integers(0, 256, 3).astype(np.uint8)
    return cols


@pytest.mark.parametrize("seed", range(5))
def test_equals_python_brute_force(seed):
    rng = np.random.default_rng(seed)
    cols = _random_cols(rng, 2000, bytes_domain=(seed % 2 == 0))
    cutoff = int(rng.integers(8000, 10600))
    got, _ = oracle.q1(cols, cutoff)
    ref = brute_q1(cols, cutoff)
    assert [(r["rf_byte"], r["ls_byte"]) for r in got] == list(ref)
    for r, a in zip(got, ref.values()):
        assert [r[k] for k in SUMS] == a
        assert r["avg_qty"] == float(Fraction(a[1], 100 * a[0]))
        assert r["avg_price"] == float(Fraction(a[2], 100 * a[0]))
        assert r["avg_disc"] == float(Fraction(a[5], 100 * a[0]))


def test_equals_pyarrow_decimal128():
    """SQL decimal semantics via pyarrow: l_extendedprice, l_discount, l_tax as
    DECIMAL(15,2); (1 - l_discount), (1 + l_tax) and the products exact."""
    pa = pytest.importorskip("pyarrow")
    pc = pytest.importorskip("pyarrow.compute")
    from decimal import Decimal
    cols = ragen.lineitem(101, ragen.rows_for_sf(0.01), ragen.parts_for_sf(0.01))
    got, status = oracle.q1(cols, CUTOFF)
    assert status == 0
    sel = cols["shipdate"] <= CUTOFF
    d152 = pa.decimal128(15, 2)
    dec = lambda a: pa.array([Decimal(int(v)).scaleb(-2) for v in a[sel]], type=d152)
    qty, price, disc, tax = (dec(cols[c]) for c in ("quantity", "extendedprice", "discount", "tax"))
    one = pa.scalar(Decimal("1.00"), type=pa.decimal128(3, 2))
    d52 = pa.decimal128(5, 2)  # 1 - discount, 1 + tax are in [0, 2]
    disc_price = pc.multiply(price, pc.subtract(one, disc).cast(d52)).cast(pa.decimal128(24, 4))
    charge = pc.multiply(disc_price, pc.add(one, tax).cast(d52))
    t = pa.table({"rf": pa.array(cols["returnflag"][sel]), "ls": pa.array(cols["linestatus"][sel]),
                  "q": qty, "p": price, "dp": disc_price, "ch": charge, "d": disc})
    agg = t.group_by(["rf", "ls"]).aggregate([("q", "sum"), ("p", "sum"), ("dp", "sum"), ("ch", "sum"),
                                              ("d", "sum"), ("rf", "count")])
    agg = agg.sort_by([("rf", "ascending"), ("ls", "ascending")]).to_pylist()
    assert len(agg) == len(got) == 4
    for r, a in zip(got, agg):
        assert (r["rf_byte"], r["ls_byte"]) == (a["rf"], a["ls"])
        assert r["count_order"] == a["rf_count"]
        assert Decimal(r["sum_qty"]).scaleb(-2) == a["q_sum"]
        assert Decimal(r["sum_base_price"]).scaleb(-2) == a["p_sum"]
        assert Decimal(r["sum_disc_price"]).scaleb(-4) == a["dp_sum"]
        assert Decimal(r["sum_charge"]).scaleb(-6) == a["ch_sum"]
        assert Decimal(r["sum_disc"]).scaleb(-2) == a["d_sum"]


def test_equals_sqlite():
    cols = ragen.lineitem(202, 200000, 20000)
    got, _ = oracle.q1(cols, CUTOFF)
    con = sqlite3.connect(":memory:")
    con.execute("create table l (sd int, rf int, ls int, q int, p int, d int, t int)")
    con.executemany("insert into l values (?,?,?,?,?,?,?)", zip(*(cols[c].tolist() for c in (
        "shipdate", "returnflag", "linestatus", "quantity", "extendedprice", "discount", "tax"))))
    res = con.execute(
        "select rf, ls, count(*), sum(q), sum(p), sum(p*(100-d)), sum(p*(100-d)*(100+t)), sum(d) "
        "from l where sd <= ? group by rf, ls order by rf, ls", (CUTOFF,)).fetchall()
    assert [(r["rf_byte"], r["ls_byte"], *[r[k] for k in SUMS]) for r in got] == [tuple(r) for r in res]


def test_invariants_and_cutoff_extremes():
    cols = ragen.lineitem(7, 100000, 2000)
    got, _ = oracle.q1(cols, CUTOFF)
    sel = cols["shipdate"] <= CUTOFF
    assert sum(r["count_order"] for r in got) == int(sel.sum())
    assert sum(r["sum_qty"] for r in got) == int(cols["quantity"][sel].sum())
    allrows, _ = oracle.q1(cols, 10561)  # >= max shipdate: every row
    assert sum(r["count_order"] for r in allrows) == cols["shipdate"].size
    none, _ = oracle.q1(cols, 8035)  # < min shipdate (8036)
    assert none == []
    # partition additivity: Q1(A u B) = Q1(A) (+) Q1(B), slotwise exact sums
    a = {k: v[:33333] for k, v in cols.items()}
    b = {k: v[33333:] for k, v in cols.items()}
    ra, _ = oracle.q1(a, CUTOFF)
    rb, _ = oracle.q1(b, CUTOFF)
    merged = {}
    for r in ra + rb:
        m = merged.setdefault((r["rf_byte"], r["ls_byte"]), [0] * len(SUMS))
        for i, k in enumerate(SUMS):
            m[i] += r[k]
    assert [[r[k] for k in SUMS] for r in got] == [merged[k] for k in sorted(merged)]


def test_statistics_match_tpch_shape():
    cols = ragen.lineitem(8, 1 << 20, 200000)
    got, _ = oracle.q1(cols, CUTOFF)
    assert [(r["returnflag"], r["linestatus"]) for r in got] == [("A", "F"), ("N", "F"), ("N", "O"), ("R", "F")]
    for r in got:
        assert abs(r["avg_qty"] - 25.5) < 0.3
        assert abs(r["avg_disc"] - 0.05) < 0.002


def test_domain_status_bits():
    cols = ragen.lineitem(9, 1000, 2000)
    _, st = oracle.q1(cols, 10561)
    assert st == 0
    bad = {k: v.copy() for k, v in cols.items()}
    bad["returnflag"][5] = ord("X")
    assert oracle.q1(bad, 10561)[1] == 1
    bad["shipdate"][5] = 20000  # not selected -> not checked
    assert oracle.q1(bad, 10561)[1] == 0
    bad2 = {k: v.copy() for k, v in cols.items()}
    bad2["discount"][3] = 101
    assert oracle.q1(bad2, 10561)[1] == 2
    bad2["discount"][3] = 100
    bad2["extendedprice"][4] = 2**31
    assert oracle.q1(bad2, 10561)[1] == 2
