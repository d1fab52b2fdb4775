"""GPU parity: libra.so's fused Q1 (+ host finalize) vs the CPU oracle.

Bit-exact: every group's count and scaled-integer sums (128-bit disc_price and
charge) and the AVG doubles (C12: one division of exact operands on both
sides), plus the domain status bits.
"""
import numpy as np
import pytest

import oracle
import ragen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
CUTOFF = 10471
KEYS = ("count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc",
        "avg_qty", "avg_price", "avg_disc")


@pytest.fixture(scope="module")
def R():
    import paper_conf_ipps_wudwcyc12_b200 as R
    return R


def to_dev(cols, offset=0):
    out = {}
    for k, v in cols.items():
        pad = np.zeros(offset, dtype=v.dtype)
        out[k] = torch.from_numpy(np.concatenate([pad, v])).cuda()[offset:]
    return out


def gpu_q1(R, dcols, cutoff=CUTOFF):
    part = R.q1(dcols, cutoff)
    torch.cuda.synchronize()
    raw = bytes(part.cpu().numpy().tobytes())
    rows, rc = R.q1_finalize(raw)
    return rows, rc, R.partials_from_bytes(raw)[0]


def assert_same(rows, exp):
    assert [(r["returnflag"], r["linestatus"]) for r in rows] == [(e["returnflag"], e["linestatus"]) for e in exp]
    for r, e in zip(rows, exp):
        for k in KEYS:
            assert r[k] == e[k], (r["returnflag"], r["linestatus"], k, r[k], e[k])


@pytest.mark.parametrize("n", [0, 1, 3, 4, 5, 255, 256, 1023, 4097, 100003])
@pytest.mark.parametrize("offset", [0, 1, 2, 3])
def test_small_sizes_and_alignment(R, n, offset):
    cols = ragen.lineitem(31 + n, n, 2000)
    exp, st = oracle.q1(cols, CUTOFF)
    rows, rc, part = gpu_q1(R, to_dev(cols, offset))
    assert rc == R.RA_OK and part.status == st == 0 and part.rows == n
    assert_same(rows, exp)


@pytest.mark.parametrize("sf", [0.01, 1.0, 10.0])
def test_scale_factors(R, sf):
    n = ragen.rows_for_sf(sf)
    cols = ragen.lineitem(3, n, ragen.parts_for_sf(sf))
    exp, st = oracle.q1(cols, CUTOFF)
    rows, rc, _ = gpu_q1(R, to_dev(cols))
    assert rc == R.RA_OK and st == 0
    assert_same(rows, exp)


@pytest.mark.parametrize("cutoff", [8035, 8036, 9298, 10000, 10471, 10561, 2**31 - 1, -(2**31)])
def test_cutoffs(R, cutoff):
    cols = ragen.lineitem(4, 200001, 20000)
    exp, _ = oracle.q1(cols, cutoff)
    rows, rc, _ = gpu_q1(R, to_dev(cols), cutoff)
    assert rc == R.RA_OK
    assert_same(rows, exp)


def test_device_generated_sf10_launch_config(R):
    """BASELINE configs[2] (SF10, 60 M rows) generated on the device exactly as
    bench.py does; oracle over the same rows regenerated on the host."""
    n = ragen.rows_for_sf(10)
    dcols = {name: torch.empty(n, dtype=getattr(torch, np.dtype(dt).name), device="cuda")
             for name, dt in ragen.LINEITEM_COLUMNS}
    ragen.lineitem_dev(3, ragen.parts_for_sf(10), dcols)
    rows, rc, _ = gpu_q1(R, dcols)
    cols = ragen.lineitem(3, n, ragen.parts_for_sf(10))
    exp, _ = oracle.q1(cols, CUTOFF)
    assert rc == R.RA_OK
    assert_same(rows, exp)


def test_sf100_full_size_launch_config(R):
    """BASELINE configs[4] at full size (SF100, 600 M rows, 22.8 GB on the
    device, seed 5 as bench.py) in bench's launch configuration (one ra_q1 over
    the whole table), plus the same rows as 4 row-range shards merged by
    ra_q1_finalize (the N=4 exchange).  Expected values: the oracle over
    50 M-row host chunks, exact sums added across chunks (partition
    additivity, pinned in test_oracle_q1), AVG = the correctly rounded exact
    quotient (C12)."""
    from fractions import Fraction
    from paper_conf_ipps_wudwcyc12_b200 import dist as rdist
    sf, seed = 100, 5
    n, parts = ragen.rows_for_sf(sf), ragen.parts_for_sf(sf)
    dcols = {name: torch.empty(n, dtype=getattr(torch, np.dtype(dt).name), device="cuda")
             for name, dt in ragen.LINEITEM_COLUMNS}
    ragen.lineitem_dev(seed, parts, dcols)
    rows, rc, part = gpu_q1(R, dcols)
    assert rc == R.RA_OK and part.rows == n
    shards = []
    for r in range(4):
        lo, hi = rdist.shard_range(n, r, 4)
        p_ = R.q1({k: v[lo:hi] for k, v in dcols.items()})
        shards.append(p_)
    torch.cuda.synchronize()
    srows, src = R.q1_finalize(b"".join(bytes(p_.cpu().numpy().tobytes()) for p_ in shards))
    del dcols
    tot = {}
    chunk = 50_000_000
    for lo in range(0, n, chunk):
        m = min(chunk, n - lo)
        part_rows, st = oracle.q1(ragen.lineitem(seed, m, parts, row0=lo), CUTOFF)
        assert st == 0
        for e in part_rows:
            g = tot.setdefault((e["returnflag"], e["linestatus"]), dict.fromkeys(
                ["count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc"], 0))
            for k in g:
                g[k] += e[k]
    exp = []
    for (rf, ls) in sorted(tot):
        g = dict(tot[(rf, ls)], returnflag=rf, linestatus=ls)
        c100 = 100 * g["count_order"]
        g["avg_qty"] = float(Fraction(g["sum_qty"], c100))
        g["avg_price"] = float(Fraction(g["sum_base_price"], c100))
        g["avg_disc"] = float(Fraction(g["sum_disc"], c100))
        exp.append(g)
    assert sum(g["sum_charge"] for g in exp) > 2**63  # SF100: Sum(charge) needs more than int64 (C11)
    assert_same(rows, exp)
    assert src == R.RA_OK
    assert_same(srows, exp)


def test_domain_errors_reported(R):
    cols = ragen.lineitem(5, 50000, 2000)
    bad = {k: v.copy() for k, v in cols.items()}
    bad["returnflag"][100] = ord("Z")
    bad["tax"][200] = 101
    exp, st = oracle.q1(bad, 10561)
    assert st == 3
    rows, rc, part = gpu_q1(R, to_dev(bad), 10561)
    assert rc == R.RA_E_DOMAIN and part.status == st
    # out-of-domain rows are not accumulated: equal to the oracle without them
    keep = np.ones(50000, bool)
    keep[[100, 200]] = False
    exp2, _ = oracle.q1({k: v[keep] for k, v in bad.items()}, 10561)
    assert_same(rows, exp2)


def test_arbitrary_bytes_random(R):
    rng = np.random.default_rng(0)
    cols = ragen.lineitem(6, 30000, 2000)
    idx = rng.integers(0, 30000, 50)
    cols["linestatus"][idx] = rng.integers(0, 256, 50).astype(np.uint8)
    exp, st = oracle.q1(cols, 10561)
    rows, rc, part = gpu_q1(R, to_dev(cols), 10561)
    assert part.status == st
    assert rc == (R.RA_E_DOMAIN if st else R.RA_OK)


def test_shard_partials_merge_exactly(R):
    """Row-range shards -> partials -> exact slotwise merge == oracle on the whole."""
    n = 1_000_003
    cols = ragen.lineitem(7, n, 200000)
    exp, _ = oracle.q1(cols, CUTOFF)
    cuts = [0, 1, 250001, 600000, n]
    raws = b""
    for a, b in zip(cuts[:-1], cuts[1:]):
        part = R.q1(to_dev({k: v[a:b] for k, v in cols.items()}), CUTOFF)
        torch.cuda.synchronize()
        raws += part.cpu().numpy().tobytes()
    rows, rc = R.q1_finalize(raws)
    assert rc == R.RA_OK
    assert_same(rows, exp)


def test_repeated_launches_self_clean(R):
    cols = ragen.lineitem(8, 300000, 20000)
    exp, _ = oracle.q1(cols, CUTOFF)
    d = to_dev(cols)
    parts = [R.q1(d, CUTOFF) for _ in range(20)]
    torch.cuda.synchronize()
    for p in parts:
        rows, rc = R.q1_finalize(bytes(p.cpu().numpy().tobytes()))
        assert_same(rows, exp)


def _widen(cols, frac, seed):
    """Put a fraction of rows at in-domain values outside the TMA kernel's
    narrow accumulators (quantity >= 2^16, price >= 2^24), plus the exact
    boundary values, so both accumulation paths and their flushes are hit."""
    rng = np.random.default_rng(seed)
    n = cols["quantity"].size
    out = {k: v.copy() for k, v in cols.items()}
    idx = rng.choice(n, int(n * frac), replace=False)
    out["quantity"][idx] = rng.integers(1 << 16, 1 << 31, idx.size)
    idx2 = rng.choice(n, int(n * frac), replace=False)
    out["extendedprice"][idx2] = rng.integers(1 << 24, 1 << 31, idx2.size)
    edges = np.array([(1 << 16) - 1, 1 << 16, (1 << 24) - 1, 1 << 24, (1 << 31) - 1, 0])
    pos = rng.choice(n, 60, replace=False)
    out["quantity"][pos[:30]] = edges[np.arange(30) % edges.size]
    out["extendedprice"][pos[30:]] = edges[np.arange(30) % edges.size]
    out["discount"][pos[::7]] = 100
    out["tax"][pos[::5]] = 100
    return out


@pytest.mark.parametrize("n,frac", [(5000, 0.2), (1_000_003, 0.01), (12_000_017, 0.001)])
def test_wide_in_domain_values(R, n, frac):
    cols = _widen(ragen.lineitem(41, n, 200000), frac, n)
    exp, st = oracle.q1(cols, 10561)
    assert st == 0
    rows, rc, part = gpu_q1(R, to_dev(cols), 10561)
    assert rc == R.RA_OK and part.status == 0
    assert_same(rows, exp)


def test_all_rows_one_group_many_tiles(R):
    """Every row in one slot at maximal narrow values: the 32-bit narrow sums
    reach their bound between flushes (count<<16|disc, price < 2^24 x 256)."""
    n = 10_000_000
    cols = ragen.lineitem(42, n, 2000)
    cols["returnflag"][:] = ord("R")
    cols["linestatus"][:] = ord("O")
    cols["quantity"][:] = (1 << 16) - 1
    cols["extendedprice"][:] = (1 << 24) - 1
    cols["discount"][:] = 100
    cols["discount"][::2] = 0
    cols["tax"][:] = 100
    exp, _ = oracle.q1(cols, 2**31 - 1)
    rows, rc, _ = gpu_q1(R, to_dev(cols), 2**31 - 1)
    assert rc == R.RA_OK
    assert_same(rows, exp)


@pytest.mark.parametrize("offsets", [(0, 1, 0, 0, 0, 0, 0), (0, 0, 0, 1, 0, 0, 0), (3, 2, 1, 0, 0, 0, 0)])
def test_columns_not_coalignable(R, offsets):
    """Column views whose 16-B alignment differs per column cannot use the
    bulk-copy kernel; the grid-stride kernel must give the same result."""
    n = 300_007
    cols = ragen.lineitem(43, n, 20000)
    exp, _ = oracle.q1(cols, CUTOFF)
    d = {}
    for (name, v), off in zip(cols.items(), offsets):
        d[name] = torch.from_numpy(np.concatenate([np.zeros(off, v.dtype), v])).cuda()[off:]
    rows, rc, _ = gpu_q1(R, d)
    assert rc == R.RA_OK
    assert_same(rows, exp)


def test_n_past_2_pow_31_closed_form(R):
    """2^31 + 2^28 identical wide rows (92 GB on the device) -- the sums are n
    times the row's values, exact, past 2^31 rows and with Sum(charge) far
    beyond int64 per group."""
    n = (1 << 31) + (1 << 28)
    vals = {"shipdate": 9000, "returnflag": ord("R"), "linestatus": ord("F"), "quantity": 5000,
            "extendedprice": 10494950, "discount": 0, "tax": 8}
    cols = {name: torch.empty(n, dtype=getattr(torch, np.dtype(dt).name), device="cuda")
            for name, dt in ragen.LINEITEM_COLUMNS}
    for k, v in vals.items():
        cols[k].fill_(v)
    rows, rc, part = gpu_q1(R, cols)
    assert rc == R.RA_OK and part.rows == n and len(rows) == 1
    r = rows[0]
    dp = 10494950 * 100
    assert (r["returnflag"], r["linestatus"]) == ("R", "F")
    assert r["count_order"] == n and r["sum_qty"] == 5000 * n and r["sum_base_price"] == 10494950 * n
    assert r["sum_disc"] == 0 and r["sum_disc_price"] == dp * n and r["sum_charge"] == dp * 108 * n
    assert r["sum_charge"] > 2**63
    # AVG per reading C12: (double)Sum / (double)(100 count)
    assert r["avg_qty"] == float(5000 * n) / float(100 * n) and r["avg_disc"] == 0.0
    assert r["avg_price"] == float(10494950 * n) / float(100 * n)
