"""Input generator: the C host implementation matches the documented recipe
(an independent numpy re-implementation) and any row range is reproducible."""
import numpy as np
import pytest

import ragen
from ragen import np_ref


@pytest.mark.parametrize("row0,n", [(0, 1), (0, 4097), (123456789, 50000), (2**33 + 5, 1000)])
def test_int32_matches_numpy_recipe(row0, n):
    a = ragen.int32_column(11, n, row0=row0)
    b = np_ref.int32_column(11, n, row0=row0)
    np.testing.assert_array_equal(a, b)


@pytest.mark.parametrize("row0,n,parts", [(0, 3, 2000), (777, 100000, 20000), (5 * 10**8, 20000, 20_000_000)])
def test_lineitem_matches_numpy_recipe(row0, n, parts):
    a = ragen.lineitem(5, n, parts, row0=row0)
    b = np_ref.lineitem(5, n, parts, row0=row0)
    for k in b:
        np.testing.assert_array_equal(a[k], b[k], err_msg=k)


def test_ranges_are_reproducible():
    whole = ragen.int32_column(3, 300000)
    part = ragen.int32_column(3, 100000, row0=150000)
    np.testing.assert_array_equal(whole[150000:250000], part)
    lw = ragen.lineitem(3, 300000, 2000)
    lp = ragen.lineitem(3, 1000, 2000, row0=299000)
    for k in lw:
        np.testing.assert_array_equal(lw[k][299000:], lp[k])


def test_int32_is_uniform():
    x = ragen.int32_column(1, 1 << 20).astype(np.int64)
    # mean of U(int32) is -0.5; sd = 2^32/sqrt(12); 6-sigma band on the mean
    sd = 2**32 / np.sqrt(12) / np.sqrt(x.size)
    assert abs(x.mean() + 0.5) < 6 * sd
    assert x.min() < -(2**31) + 2**22 and x.max() > 2**31 - 2**22


def test_lineitem_marginals_match_tpch_shape():
    """SURVEY A.4 simulated marginals of the C15 rules (10 M rows):
    selected 0.98593; A-F .2469, N-F .0064, N-O .4859, R-F .2467."""
    n = 1 << 21
    li = ragen.lineitem(9, n, 200000)
    sel = li["shipdate"] <= 10471
    assert abs(sel.mean() - 0.98593) < 0.002
    key = li["returnflag"].astype(np.int32) * 256 + li["linestatus"]
    for (rf, ls), frac in {("A", "F"): .2469, ("N", "F"): .0064, ("N", "O"): .4859, ("R", "F"): .2467}.items():
        f = (sel & (key == ord(rf) * 256 + ord(ls))).mean()
        assert abs(f - frac) < 0.003, (rf, ls, f)
    assert li["quantity"].min() == 100 and li["quantity"].max() == 5000
    assert li["discount"].min() == 0 and li["discount"].max() == 10
    assert li["tax"].min() == 0 and li["tax"].max() == 8
    assert li["shipdate"].min() >= 8036 and li["shipdate"].max() <= 10561


def test_nested_thresholds_fractions():
    """s=.5 -> .4997/.2500/.1248 on 2^22 samples; exact fractions s^j."""
    x = ragen.int32_column(2, 1 << 22)
    for s in (0.01, 0.5, 0.9):
        ts = ragen.nested_thresholds(s, 3)
        for j, t in enumerate(ts):
            f = (x < t).mean()
            p = s ** (j + 1)
            assert abs(f - p) < 6 * np.sqrt(p * (1 - p) / x.size) + 1e-9, (s, j, f)
