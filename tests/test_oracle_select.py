"""Pins for the oracle's SELECT / SELECT-chain / fission definitions.

Each check ties oracle/oracle.c to something other than itself: the paper's
Table I example, a pure-Python list comprehension (brute force), numpy boolean
indexing (a library routine with the same stable semantics), closed-form
invariants (selectivity 0/1, 50%·50% = 25%, fused == unfused, chunking and
partition additivity).
"""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
import ragen
from golden_io import table1_select

I32 = st.integers(min_value=-(2**31), max_value=2**31 - 1)
OPS = ["lt", "le", "gt", "ge", "eq", "ne"]
PY_CMP = {
    "lt": lambda x, v: x < v, "le": lambda x, v: x <= v, "gt": lambda x, v: x > v,
    "ge": lambda x, v: x >= v, "eq": lambda x, v: x == v, "ne": lambda x, v: x != v,
}


def brute(xs, preds):
    return [x for x in xs if all(PY_CMP[op](x, v) for op, v in preds)]


def test_table1_select_example():
    x, preds, expect = table1_select()
    assert oracle.select(x, preds).tolist() == expect


@settings(max_examples=300, deadline=None)
@given(xs=st.lists(st.one_of(I32, st.integers(-5, 5)), max_size=60),
       preds=st.lists(st.tuples(st.sampled_from(OPS), st.one_of(I32, st.integers(-5, 5))), max_size=8))
def test_select_equals_brute_force(xs, preds):
    assert oracle.select(xs, preds).tolist() == brute(xs, preds)
    assert oracle.select(xs, preds, fused=False).tolist() == brute(xs, preds)
    assert oracle.select_count(xs, preds) == len(brute(xs, preds))


@settings(max_examples=100, deadline=None)
@given(xs=st.lists(st.integers(-4, 4), max_size=40),
       preds=st.lists(st.tuples(st.sampled_from(OPS), st.integers(-4, 4)), max_size=4),
       chunk=st.integers(1, 50))
def test_chunked_equals_brute_force(xs, preds, chunk):
    assert oracle.select_chunked(xs, preds, chunk).tolist() == brute(xs, preds)


def test_select_equals_numpy_mask():
    x = ragen.int32_column(1, 1 << 18)
    preds = [("gt", -(10**9)), ("lt", 10**9), ("ne", int(x[17])), ("le", 2**30)]
    m = (x > -(10**9)) & (x < 10**9) & (x != x[17]) & (x <= 2**30)
    np.testing.assert_array_equal(oracle.select(x, preds), x[m])


def test_selectivity_zero_and_one():
    """LT INT32_MIN selects nothing; GE INT32_MIN and k=0 are identity."""
    x = ragen.int32_column(4, 100003)
    assert oracle.select(x, [("lt", -(2**31))]).size == 0
    np.testing.assert_array_equal(oracle.select(x, [("ge", -(2**31))]), x)
    np.testing.assert_array_equal(oracle.select(x, []), x)
    assert oracle.select([], [("lt", 0)]).size == 0


def test_two_fifty_percent_selects_keep_a_quarter():
    """"two back-to-back SELECTs keep 25% of the original data"."""
    n = 1 << 22
    x = ragen.int32_column(2, n)
    t = ragen.nested_thresholds(0.5, 2)
    preds = [("lt", t[0]), ("lt", t[1])]
    c1 = oracle.select_count(x, preds[:1])
    c2 = oracle.select_count(x, preds)
    for c, p in ((c1, 0.5), (c2, 0.25)):
        assert abs(c - p * n) < 6 * np.sqrt(n * p * (1 - p))


@pytest.mark.parametrize("s,k", [(0.01, 2), (0.5, 3), (0.9, 2), (0.25, 1)])
def test_fused_equals_unfused_and_chunks(s, k):
    """Fused chain == unfused composition (L580-581); fission chunks CPU-gathered
    in order == device result (L1466-1468); row-range shards concatenate."""
    x = ragen.int32_column(5, 300001)
    preds = [("lt", t) for t in ragen.nested_thresholds(s, k)]
    fused = oracle.select(x, preds)
    np.testing.assert_array_equal(oracle.select(x, preds, fused=False), fused)
    for chunk in (1, 4095, 65536, 300001, 10**7):
        np.testing.assert_array_equal(oracle.select_chunked(x, preds, chunk), fused)
    cuts = [0, 7, 100000, 233333, x.size]
    shards = [oracle.select(x[a:b], preds) for a, b in zip(cuts[:-1], cuts[1:])]
    np.testing.assert_array_equal(np.concatenate(shards), fused)


def test_invalid_op_rejected():
    with pytest.raises(ValueError):
        oracle.select([1, 2], [(9, 0)])


# ---------------------------------------------------------------- tuples (f3)
def test_table1_tuple_select_and_project():
    """Table I: select [field.0==2] x -> (2,False,b); project [0,2] x -> {(3,a),(4,a),(2,b)}."""
    from golden_io import table1_tuples
    cols, sel, sel_out, proj_fields, proj_out = table1_tuples()
    f = [np.array(c, dtype=np.int32) for c in cols]
    rowids, outs = oracle.select_rows(f[0], [sel], f)
    assert rowids.tolist() == [2]
    assert tuple(int(o[0]) for o in outs) == sel_out
    rowids, outs = oracle.select_rows(f[0], [], [f[j] for j in proj_fields])  # k = 0: PROJECT
    assert rowids.tolist() == [0, 1, 2]
    assert list(zip(*[o.tolist() for o in outs])) == proj_out


@settings(max_examples=200, deadline=None)
@given(rows=st.lists(st.tuples(st.one_of(I32, st.integers(-4, 4)), I32, st.integers(-2**63, 2**63 - 1)),
                     max_size=50),
       preds=st.lists(st.tuples(st.sampled_from(OPS), st.one_of(I32, st.integers(-4, 4))), max_size=4))
def test_select_rows_equals_brute_force(rows, preds):
    key = np.array([r[0] for r in rows], dtype=np.int32)
    a = np.array([r[1] for r in rows], dtype=np.int32)
    b = np.array([r[2] for r in rows], dtype=np.int64)
    exp = [(i, r[1], r[2]) for i, r in enumerate(rows) if all(PY_CMP[op](r[0], v) for op, v in preds)]
    rowids, (oa, ob) = oracle.select_rows(key, preds, [a, b])
    assert list(zip(rowids.tolist(), oa.tolist(), ob.tolist())) == exp


def test_select_rows_matches_numpy_and_value_select():
    x = ragen.int32_column(9, 100_003)
    pay = np.arange(x.size, dtype=np.int64) * 7 - 3
    preds = [("gt", -(2**30)), ("lt", 2**29), ("ne", int(x[17]))]
    mask = (x > -(2**30)) & (x < 2**29) & (x != x[17])
    rowids, (okey, opay) = oracle.select_rows(x, preds, [x, pay])
    assert np.array_equal(rowids, np.flatnonzero(mask))
    assert np.array_equal(okey, x[mask]) and np.array_equal(opay, pay[mask])
    assert np.array_equal(okey, oracle.select(x, preds))


# ----------------------------------------------------- several SELECTs (f2)
@settings(max_examples=200, deadline=None)
@given(xs=st.lists(st.one_of(I32, st.integers(-5, 5)), max_size=60),
       chains=st.lists(st.lists(st.tuples(st.sampled_from(OPS), st.one_of(I32, st.integers(-5, 5))), max_size=4),
                       min_size=1, max_size=4))
def test_select_multi_equals_brute_force_per_output(xs, chains):
    outs = oracle.select_multi(xs, chains)
    assert [o.tolist() for o in outs] == [brute(xs, c) for c in chains]


def test_select_multi_numpy_and_disjoint_cover():
    """Two complementary SELECTs (x < t, x >= t) partition the input: the
    outputs' sizes add to n, and each equals numpy boolean indexing."""
    x = ragen.int32_column(10, 200_001)
    t = int(x[123])
    lo, hi = oracle.select_multi(x, [[("lt", t)], [("ge", t)]])
    assert np.array_equal(lo, x[x < t]) and np.array_equal(hi, x[x >= t])
    assert lo.size + hi.size == x.size
