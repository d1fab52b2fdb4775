"""GPU parity: Q1 under kernel fission (ra_q1_fission_run).

Host-resident pinned lineitem columns streamed in chunks over several streams;
the merged partial must equal the oracle over the whole table bit for bit
(partition additivity of exact integer sums) and equal the device-resident
ra_q1 partial byte for byte.
"""
import ctypes

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


def pinned(cols):
    return {k: torch.from_numpy(v).pin_memory() for k, v in cols.items()}


def streams(S):
    return [torch.cuda.Stream() for _ in range(S)]


def assert_same(rows, exp):
    assert [(r["returnflag"], r["linestatus"]) for r in rows] == [(e["returnflag"], e["linestatus"]) for e in exp]
    for r, e in zip(rows, exp):
        for k in KEYS:
            assert r[k] == e[k], (r["returnflag"], r["linestatus"], k, r[k], e[k])


@pytest.mark.parametrize("n,chunk", [(0, 1000), (1, 1000), (5, 2), (100003, 4096), (100003, 100003),
                                     (100003, 1 << 20), ((1 << 20) + 7, 1 << 16), ((1 << 20) + 7, 333333)])
@pytest.mark.parametrize("S", [1, 2, 3])
def test_fission_matches_oracle(R, n, chunk, S):
    cols = ragen.lineitem(41 + n, n, 20000)
    exp, st = oracle.q1(cols, CUTOFF)
    part = R.q1_fission_run(pinned(cols), chunk, streams(S))
    assert part.status == st == 0 and part.rows == n and part.n_groups == 6
    rows, rc = R.q1_finalize(bytes(part))
    assert rc == R.RA_OK
    assert_same(rows, exp)


def test_fission_equals_device_partial(R):
    n = ragen.rows_for_sf(1)
    cols = ragen.lineitem(7, n, ragen.parts_for_sf(1))
    dev = R.q1({k: torch.from_numpy(v).cuda() for k, v in cols.items()}, CUTOFF)
    torch.cuda.synchronize()
    part = R.q1_fission_run(pinned(cols), 1 << 22, streams(3))
    assert bytes(part) == bytes(dev.cpu().numpy().tobytes())


def test_fission_domain_error_in_one_chunk(R):
    n = 50000
    cols = ragen.lineitem(8, n, 20000)
    sel = np.nonzero(cols["shipdate"] <= CUTOFF)[0]
    cols["returnflag"][sel[-1]] = ord("X")  # last chunk only
    _, st = oracle.q1(cols, CUTOFF)
    part = R.q1_fission_run(pinned(cols), 4096, streams(3))
    assert part.status == st and part.status & 1
    _, rc = R.q1_finalize(bytes(part))
    assert rc == R.RA_E_DOMAIN


def test_fission_rejects_pageable(R):
    cols = ragen.lineitem(9, 1000, 2000)
    h = pinned(cols)
    h["tax"] = torch.from_numpy(cols["tax"])  # pageable
    with pytest.raises(ValueError):
        R.q1_fission_run(h, 256, streams(2))
    # through the raw C ABI the library itself refuses it
    ws = torch.zeros(R.ra_q1_fission_workspace_bytes(256, 1), dtype=torch.uint8, device="cuda")
    st = (ctypes.c_void_p * 1)(torch.cuda.current_stream().cuda_stream)
    with pytest.raises(R.RAError) as e:
        R.ra_q1_fission_run(R.lineitem_struct(h), 1000, CUTOFF, 256, st, 1, R.ra_q1_partial(),
                            ws.data_ptr(), ws.numel())
    assert e.value.code == R.RA_E_NOT_PINNED


def test_first_call_on_a_fresh_workspace(R):
    """The workspace helper zero-fills a new workspace on the current stream;
    the fission runtimes then use it from their own streams.  Every first call
    on a fresh workspace must see the fill complete (regression test)."""
    n = 3_000_000
    cols = ragen.lineitem(21, n, 20000)
    exp, _ = oracle.q1(cols, R.Q1_CUTOFF_DELTA90)
    h = {k: torch.from_numpy(v).pin_memory() for k, v in cols.items()}
    streams = [torch.cuda.Stream() for _ in range(3)]
    for _ in range(6):
        R._WS.clear()
        torch.cuda.synchronize()
        rows, rc = R.q1_finalize(bytes(R.q1_fission_run(h, 1 << 19, streams)))
        assert rc == R.RA_OK
        assert [(r["returnflag"], r["linestatus"], r["count_order"], r["sum_charge"]) for r in rows] == \
               [(e["returnflag"], e["linestatus"], e["count_order"], e["sum_charge"]) for e in exp]


def test_bench_configuration_fresh_workspaces(R):
    """Round 1 saw one bench run whose wide and narrow Q1-fission results
    disagreed on first calls on fresh workspaces.  Root cause: the workspace's
    zero fill ran on the current stream while the fission streams (not ordered
    after it) had already accumulated chunk partials into the same bytes.
    bench.py's exact configuration (SF10, wide chunk 2^22 / narrow chunk 2^23,
    3 streams), a fresh workspace before each of 20 iterations and no host
    synchronisation in between: every result equals the oracle."""
    sf = 10
    n = ragen.rows_for_sf(sf)
    cols = ragen.lineitem(5, n, ragen.parts_for_sf(sf))
    exp, st = oracle.q1(cols, CUTOFF)
    assert st == 0
    h = pinned(cols)
    dcols = {k: v.cuda() for k, v in h.items()}
    enc, est = R.q1_encode(dcols)
    assert int(est.item()) == 0
    del dcols
    hn = {k: v.cpu().pin_memory() for k, v in enc.items()}
    del enc
    ss = streams(3)
    for it in range(20):
        R._WS.clear()
        rows, rc = R.q1_finalize(bytes(R.q1_fission_run(h, 1 << 22, ss)))
        assert rc == R.RA_OK
        assert_same(rows, exp)
        R._WS.clear()
        nrows, nrc = R.q1_finalize(bytes(R.q1_narrow_fission_run(hn, 1 << 23, ss)))
        assert nrc == R.RA_OK
        assert_same(nrows, exp)
