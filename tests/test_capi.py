"""C-ABI checks that need no GPU: libra.so loads, exports every entry point
include/ra.h declares, sizes workspaces, rejects bad arguments before touching
CUDA, and its host-side Q1 finalize merges partials exactly (fed with partials
assembled from the oracle's exact group sums)."""
import ctypes
import subprocess

import numpy as np
import pytest

import oracle
import ragen

R = pytest.importorskip("paper_conf_ipps_wudwcyc12_b200")


def test_exports_every_header_symbol():
    declared = R.exported_symbols_from_header()
    assert len(declared) >= 12
    nm = subprocess.run(["nm", "-D", "--defined-only", R.LIB_PATH], capture_output=True, text=True).stdout
    exported = {line.split()[-1] for line in nm.splitlines() if " T " in line}
    assert set(declared) <= exported, set(declared) - exported
    assert {s for s in exported if s.startswith("ra_")} == set(declared)


def test_struct_sizes_match_header_layout():
    assert ctypes.sizeof(R.ra_pred) == 8
    assert ctypes.sizeof(R.ra_q1_group) == 64
    assert ctypes.sizeof(R.ra_q1_partial) == 16 + 6 * 64
    assert ctypes.sizeof(R.ra_q1_row) == 8 + 8 * 8 + 3 * 8
    assert ctypes.sizeof(R.ra_lineitem_narrow) == ctypes.sizeof(R.ra_lineitem_narrow_out) == 6 * 8
    assert R.ra_version() == 1


def test_workspace_sizes():
    assert R.ra_select_workspace_bytes(0, 1, 1) >= 256
    f = R.ra_select_workspace_bytes(1 << 28, 2, 1)
    u = R.ra_select_workspace_bytes(1 << 28, 2, 0)
    assert f < 2 << 20  # status words only: ~16 B per 4096-row tile
    assert u >= f + 2 * 4 * (1 << 28)  # two device-resident intermediates
    assert R.ra_select_workspace_bytes(1 << 28, 1, 0) == f  # k=1 never materialises
    assert R.ra_fission_workspace_bytes(1 << 20, 3, 2, 1) >= 3 * 2 * 4 * (1 << 20)
    assert R.ra_fission_workspace_bytes(0, 3, 2, 1) == 0
    # several outputs: status words only, two per 8192-row tile at most (M = 3, 4)
    m = R.ra_select_multi_workspace_bytes(1 << 28)
    assert 16 * ((1 << 28) // 8192) <= m <= 16 * ((1 << 28) // 8192 + 2) + 512
    assert R.ra_select_multi_workspace_bytes(1 << 10) < R.ra_select_multi_workspace_bytes(1 << 20) <= m
    # tuple SELECT: status words + order masks (n/8 + n/170 B) + id staging (4 B/row)
    t = R.ra_select_rows_workspace_bytes(1 << 28, 2)
    assert t >= f + (1 << 28) // 8 + 4 * (1 << 28)


def test_argument_errors_without_gpu():
    P = R.make_preds([("lt", 0)])
    with pytest.raises(R.RAError) as e:  # null count
        R.ra_select_chain(0, 10, P, 1, 1, 0, 10, 0, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError) as e:  # k > 8
        R.ra_select_chain(0, 0, R.make_preds([("lt", 0)] * 9), 9, 1, 0, 0, 8, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError) as e:  # workspace too small
        R.ra_select_chain(4096, 1 << 20, P, 1, 1, 4096, 1 << 20, 8, 256, 16, 0)
    assert e.value.code == R.RA_E_WORKSPACE
    with pytest.raises(R.RAError) as e:  # misaligned
        R.ra_select_chain(4098, 10, P, 1, 1, 4096, 10, 8, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError) as e:  # bad op
        R.ra_select_chain(4096, 10, R.make_preds([(17, 0)]), 1, 1, 4096, 10, 8, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    li = R.ra_lineitem()
    with pytest.raises(R.RAError) as e:  # null columns
        R.ra_q1(li, 5, 10471, 4096, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError) as e:  # n >= 2^32
        R.ra_q1(li, 1 << 32, 10471, 4096, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    assert "n=" in R.ra_last_error()
    nl = R.ra_lineitem_narrow()
    with pytest.raises(R.RAError) as e:  # null narrow columns
        R.ra_q1_narrow(nl, 5, 10471, 4096, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    nl = R.ra_lineitem_narrow(*([4096 + 8] * 6))
    with pytest.raises(R.RAError) as e:  # narrow columns not 16-B aligned
        R.ra_q1_narrow(nl, 5, 10471, 4096, 256, 1 << 20, 0)
    assert e.value.code == R.RA_E_INVAL
    nl = R.ra_lineitem_narrow(*([4096] * 6))
    with pytest.raises(R.RAError) as e:  # workspace too small
        R.ra_q1_narrow(nl, 5, 10471, 4096, 256, 16, 0)
    assert e.value.code == R.RA_E_WORKSPACE
    with pytest.raises(R.RAError) as e:  # encode: null output columns
        R.ra_q1_encode(R.ra_lineitem(*([4096] * 7)), 5, R.ra_lineitem_narrow_out(), 4096, 0)
    assert e.value.code == R.RA_E_INVAL


SLOT = {(ord(rf), ord(ls)): 2 * i + j for i, rf in enumerate("ANR") for j, ls in enumerate("FO")}


def partial_from_oracle_rows(rows, status=0, nrows=0):
    p = R.ra_q1_partial()
    p.status, p.n_groups, p.rows = status, 6, nrows
    for r in rows:
        g = p.group[SLOT[(r["rf_byte"], r["ls_byte"])]]
        g.count, g.sum_qty, g.sum_base_price, g.sum_disc = (
            r["count_order"], r["sum_qty"], r["sum_base_price"], r["sum_disc"])
        g.sum_disc_price_lo, g.sum_disc_price_hi = r["sum_disc_price"] & (2**64 - 1), r["sum_disc_price"] >> 64
        g.sum_charge_lo, g.sum_charge_hi = r["sum_charge"] & (2**64 - 1), r["sum_charge"] >> 64
    return p


def test_finalize_merges_shards_exactly():
    cols = ragen.lineitem(12, 400000, 200000)
    whole, _ = oracle.q1(cols, 10471)
    cuts = [0, 100, 150000, 400000]
    parts = (R.ra_q1_partial * 3)()
    for i, (a, b) in enumerate(zip(cuts[:-1], cuts[1:])):
        rows, _ = oracle.q1({k: v[a:b] for k, v in cols.items()}, 10471)
        parts[i] = partial_from_oracle_rows(rows)
    got, rc = R.q1_finalize(parts)
    assert rc == R.RA_OK
    assert len(got) == len(whole) == 4
    for g, w in zip(got, whole):
        for k in ("count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc",
                  "avg_qty", "avg_price", "avg_disc"):
            assert g[k] == w[k], k


def test_finalize_128bit_charge_and_domain():
    p = R.ra_q1_partial()
    p.group[3].count = 5
    p.group[3].sum_charge_lo, p.group[3].sum_charge_hi = 2**64 - 1, 0
    q = R.ra_q1_partial()
    q.group[3].count = 1
    q.group[3].sum_charge_lo = 1
    q.status = 2
    got, rc = R.q1_finalize((R.ra_q1_partial * 2)(p, q))
    assert rc == R.RA_E_DOMAIN
    assert got[0]["sum_charge"] == 2**64 and got[0]["count_order"] == 6
    assert (got[0]["returnflag"], got[0]["linestatus"]) == ("N", "O")


def _multi_args(M, n=100, outs=None, caps=None, cnts=None, ks=None, chains=None, ws=256, wsb=1 << 20, d_in=4096):
    import ctypes
    keep = [R.make_preds([("lt", 0)]) for _ in range(max(1, M))]
    ch = (ctypes.c_void_p * max(1, M))(*(chains if chains is not None else [ctypes.addressof(p) for p in keep]))
    k = (ctypes.c_int * max(1, M))(*(ks if ks is not None else [1] * M))
    op = (ctypes.c_void_p * max(1, M))(*(outs if outs is not None else [8192] * M))
    cp = (ctypes.c_int64 * max(1, M))(*(caps if caps is not None else [n] * M))
    cn = (ctypes.c_void_p * max(1, M))(*(cnts if cnts is not None else [16384 + 8 * o for o in range(M)]))
    return (d_in, n, ch, k, M, op, cp, cn, ws, wsb, 0), keep


@pytest.mark.parametrize("case", ["M0", "M5", "null_ws", "misaligned_in", "misaligned_out", "misaligned_count",
                                  "negative_cap", "k9", "bad_op", "null_chain", "small_ws", "huge_n"])
def test_select_multi_argument_errors_without_gpu(case):
    """ra_select_multi rejects bad arguments before touching CUDA."""
    kw = {"M0": dict(M=0), "M5": dict(M=5), "null_ws": dict(M=2, ws=0), "misaligned_in": dict(M=2, d_in=4098),
          "misaligned_out": dict(M=2, outs=[8192, 8194]), "misaligned_count": dict(M=2, cnts=[16384, 16388]),
          "negative_cap": dict(M=2, caps=[10, -1]), "k9": dict(M=1, ks=[9]), "null_chain": dict(M=2, chains=[0, 0]),
          "small_ws": dict(M=3, n=1 << 24, wsb=4096), "huge_n": dict(M=1, n=1 << 34, wsb=1 << 40)}
    if case == "bad_op":
        import ctypes
        bad = R.make_preds([(17, 0)])
        args, keep = _multi_args(1, chains=[ctypes.addressof(bad)])
    else:
        args, keep = _multi_args(**kw[case])
    with pytest.raises(R.RAError) as e:
        R.ra_select_multi(*args)
    assert e.value.code == (R.RA_E_WORKSPACE if case == "small_ws" else R.RA_E_INVAL), (case, R.ra_last_error())


def test_select_offsets_argument_errors_without_gpu():
    for bad in (0, -3, R.RA_MAX_RANKS + 1):
        with pytest.raises(R.RAError) as e:
            R.ra_select_offsets(4096, bad, 8192, 16384, 0)
        assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError) as e:  # no output at all
        R.ra_select_offsets(4096, 4, 0, 0, 0)
    assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError) as e:  # misaligned
        R.ra_select_offsets(4100, 4, 8192, 0, 0)
    assert e.value.code == R.RA_E_INVAL
