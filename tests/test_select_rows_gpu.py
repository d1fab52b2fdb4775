"""GPU parity of the tuple SELECT (ra_select_rows) through the
C-ABI against the CPU oracle (oracle.select_rows): row ids and every payload
field of the selected rows, bit-exact, in input order; Table I's SELECT and
PROJECT examples; ragged/misaligned key views, many tiles, capacity limits."""
import numpy as np
import pytest

import oracle
import ragen
from golden_io import table1_tuples

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def R():
    import paper_conf_ipps_wudwcyc12_b200 as R
    return R


def check(R, key, preds, payloads, offset=0, rowids=True):
    kd = torch.from_numpy(np.concatenate([np.zeros(offset, np.int32), key])).cuda()[offset:]
    pd = [torch.from_numpy(p).cuda() for p in payloads]
    ids, outs, cnt = R.select_rows(kd, preds, pd, rowids=rowids)
    torch.cuda.synchronize()
    c = int(cnt.item())
    exp_ids, exp_outs = oracle.select_rows(key, preds, payloads)
    assert c == exp_ids.size
    if rowids:
        assert np.array_equal(ids[:c].cpu().numpy().astype(np.int64), exp_ids)
    for o, e in zip(outs, exp_outs):
        assert np.array_equal(o[:c].cpu().numpy(), e)


def test_table1_examples(R):
    cols, sel, sel_out, proj_fields, proj_out = table1_tuples()
    f = [np.array(c, dtype=np.int32) for c in cols]
    fd = [torch.from_numpy(c).cuda() for c in f]
    ids, outs, cnt = R.select_rows(fd[0], [sel], fd)
    torch.cuda.synchronize()
    assert int(cnt.item()) == 1 and ids[0].item() == 2
    assert tuple(int(o[0].item()) for o in outs) == sel_out
    ids, outs, cnt = R.select_rows(fd[0], [], [fd[j] for j in proj_fields])  # k = 0: PROJECT
    torch.cuda.synchronize()
    assert int(cnt.item()) == 3
    assert list(zip(*[o[:3].cpu().tolist() for o in outs])) == proj_out


@pytest.mark.parametrize("n", [0, 1, 4, 8191, 8192, 8193, 3 * 8192 + 123, 1_000_003])
@pytest.mark.parametrize("offset", [0, 1, 3])
def test_sizes_offsets(R, n, offset):
    key = ragen.int32_column(61 + n, n)
    pay4 = (np.arange(n, dtype=np.int32) * 3 + 1)
    pay8 = np.arange(n, dtype=np.int64) * (1 << 33) - 5
    check(R, key, [("lt", 0), ("gt", -(2**30))], [pay4, pay8, key], offset)
    check(R, key, [("lt", -(2**31) + 2**26)], [pay4, pay8], offset, rowids=False)  # sparse, no ids


@pytest.mark.parametrize("s,k", [(0.0, 1), (0.01, 1), (0.5, 2), (0.9, 1), (1.0, 1)])
def test_selectivities_many_tiles(R, s, k):
    n = (1 << 22) + 77
    key = ragen.int32_column(62, n)
    preds = [("ge", -(2**31))] if s == 1.0 else [("lt", -(2**31))] if s == 0.0 else \
        [("lt", t) for t in ragen.nested_thresholds(s, k)]
    pay = ragen.int32_column(63, n)
    check(R, key, preds, [pay, pay.astype(np.int64) * 11])


def test_rowids_only_and_payload_only(R):
    n = 500_000
    key = ragen.int32_column(64, n)
    kd = torch.from_numpy(key).cuda()
    exp_ids, (exp_k,) = oracle.select_rows(key, [("lt", 12345)], [key])
    ids, outs, cnt = R.select_rows(kd, [("lt", 12345)], [], rowids=True)
    torch.cuda.synchronize()
    assert np.array_equal(ids[:int(cnt.item())].cpu().numpy().astype(np.int64), exp_ids)
    ids, outs, cnt = R.select_rows(kd, [("lt", 12345)], [kd], rowids=False)
    torch.cuda.synchronize()
    assert ids is None and np.array_equal(outs[0][:int(cnt.item())].cpu().numpy(), exp_k)
    # the key gathered as a payload equals the value SELECT
    assert np.array_equal(exp_k, oracle.select(key, [("lt", 12345)]))


def test_capacity_truncates_but_counts(R):
    n = 200_000
    key = ragen.int32_column(65, n)
    kd = torch.from_numpy(key).cuda()
    exp_ids, _ = oracle.select_rows(key, [("lt", 0)], [])
    cap = 1000
    ids, outs, cnt = R.select_rows(kd, [("lt", 0)], [kd], out_cap=cap)
    torch.cuda.synchronize()
    assert int(cnt.item()) == exp_ids.size
    assert np.array_equal(ids[:cap].cpu().numpy().astype(np.int64), exp_ids[:cap])
    assert np.array_equal(outs[0][:cap].cpu().numpy(), key[exp_ids[:cap]])


@pytest.mark.parametrize("koff,poff", [(0, 0), (1, 1), (3, 3), (2, 0), (0, 3), (1, 2)])
def test_payload_alignment_phases(R, koff, poff):
    """Payload columns whose 16-B phase equals the key's take 128-bit loads,
    the others element loads; both place every field exactly."""
    n = 24 * 8192 + 1001
    key = ragen.int32_column(66, n)
    p4 = ragen.int32_column(67, n)
    p8 = p4.astype(np.int64) * 7 + 1

    def dev(a, off):
        return torch.from_numpy(np.concatenate([np.zeros(off, a.dtype), a])).cuda()[off:]
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    ids, outs, cnt = R.select_rows(dev(key, koff), preds, [dev(p4, poff), dev(p8, poff), dev(key, poff)])
    torch.cuda.synchronize()
    c = int(cnt.item())
    exp_ids, exp = oracle.select_rows(key, preds, [p4, p8, key])
    assert c == exp_ids.size
    assert np.array_equal(ids[:c].cpu().numpy().astype(np.int64), exp_ids)
    for o, e in zip(outs, exp):
        assert np.array_equal(o[:c].cpu().numpy(), e)


@pytest.mark.parametrize("cap", [1, 777, 8192 * 3 + 5])
def test_capacity_never_writes_past_cap(R, cap):
    n = 300_000
    key = ragen.int32_column(68, n)
    pay = (np.arange(n, dtype=np.int64) << 20) + 3
    kd, pd = torch.from_numpy(key).cuda(), torch.from_numpy(pay).cuda()
    preds = [("gt", -(2**30))]
    exp_ids, (exp,) = oracle.select_rows(key, preds, [pay])
    ids = torch.full((cap + 64,), 0xABCDEF, dtype=torch.int32, device="cuda")
    out = torch.full((cap + 64,), -9, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    pl = (R.ra_payload * 1)()
    pl[0].col, pl[0].out, pl[0].elem_bytes = pd.data_ptr(), out.data_ptr(), 8
    wsb = R.ra_select_rows_workspace_bytes(n, 1)
    ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
    R.ra_select_rows(kd.data_ptr(), n, R.make_preds(preds), 1, ids.data_ptr(), pl, 1, cap, cnt.data_ptr(),
                     ws.data_ptr(), wsb, 0)
    torch.cuda.synchronize()
    assert int(cnt.item()) == exp_ids.size
    assert np.array_equal(ids[:cap].cpu().numpy().astype(np.int64), exp_ids[:cap])
    assert np.array_equal(out[:cap].cpu().numpy(), exp[:cap])
    assert (ids[cap:].cpu().numpy() == 0xABCDEF).all() and (out[cap:].cpu().numpy() == -9).all()


@pytest.mark.parametrize("s", [0.03, 0.05, 0.1, 0.25, 0.6])
@pytest.mark.parametrize("force_gather", [False, True])
def test_both_payload_paths(R, s, force_gather, monkeypatch):
    """The device picks the id gather (sparse) or the streaming compaction
    (dense) from the count; RA_TUPLE_GATHER forces the gather.  Both are exact
    for 4- and 8-byte fields, at selectivities on either side of the switch."""
    if force_gather:
        monkeypatch.setenv("RA_TUPLE_GATHER", "1")
    else:
        monkeypatch.delenv("RA_TUPLE_GATHER", raising=False)
    n = 40 * 8192 + 4321
    key = ragen.int32_column(69, n)
    p4 = ragen.int32_column(70, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(s, 1)]
    # without ids the sparse path takes the first n/32 from the key pass and
    # rebuilds the rest from the masks (ids_kernel): s = .05 / .1 use both
    for rowids in (True, False):
        check(R, key, preds, [p4, key], rowids=rowids)  # 4-byte fields only
        check(R, key, preds, [p4.astype(np.int64) * 5 - 7, p4], rowids=rowids)  # with an 8-byte field
        check(R, key, preds, [p4, key], offset=3, rowids=rowids)  # misaligned key view


@pytest.mark.parametrize("cap", [0, 1, 5000, 20000, 60000])
def test_capacity_without_ids_sparse(R, cap):
    """No caller ids, sparse (count between n/32 and n/12): the key pass stages
    min(out_cap, n/32) ids and ids_kernel the rest; the fields are exact up to
    out_cap and nothing is written past it."""
    n = 100 * 8192 + 77
    key = ragen.int32_column(71, n)
    p4 = ragen.int32_column(72, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(0.06, 1)]
    exp_ids, (exp,) = oracle.select_rows(key, preds, [p4])
    assert n // 32 < exp_ids.size < n // 12
    kd, pd = torch.from_numpy(key).cuda(), torch.from_numpy(p4).cuda()
    out = torch.full((cap + 64,), -9, dtype=torch.int32, device="cuda")
    pl = (R.ra_payload * 1)()
    pl[0].col, pl[0].out, pl[0].elem_bytes = pd.data_ptr(), out.data_ptr(), 4
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    wsb = R.ra_select_rows_workspace_bytes(n, 1)
    ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
    R.ra_select_rows(kd.data_ptr(), n, R.make_preds(preds), 1, 0, pl, 1, cap, cnt.data_ptr(),
                     ws.data_ptr(), wsb, int(torch.cuda.current_stream().cuda_stream))
    torch.cuda.synchronize()
    assert int(cnt.item()) == exp_ids.size
    m = min(cap, exp_ids.size)
    assert np.array_equal(out[:m].cpu().numpy(), exp[:m])
    assert (out[m:].cpu().numpy() == -9).all()


def test_argument_errors(R):
    kd = torch.zeros(16, dtype=torch.int32, device="cuda")
    bad = torch.zeros(16, dtype=torch.int16, device="cuda")
    with pytest.raises(ValueError):
        R.select_rows(kd, [("lt", 0)], [bad])
    pl = (R.ra_payload * 1)()
    pl[0].col, pl[0].out, pl[0].elem_bytes = kd.data_ptr(), kd.data_ptr(), 2
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    ws = torch.zeros(1 << 20, dtype=torch.uint8, device="cuda")
    with pytest.raises(R.RAError) as e:
        R.ra_select_rows(kd.data_ptr(), 16, R.make_preds([("lt", 0)]), 1, 0, pl, 1, 16, cnt.data_ptr(),
                         ws.data_ptr(), ws.numel(), 0)
    assert e.value.code == R.RA_E_INVAL


def test_full_size_bench_config(R):
    """bench.py's f3 leg at full size: 2^28-row key (seed 2) + two int32 fields
    (seeds 102, 103) + the key as a third field, k=2, s=.5/stage (the dense
    compaction path), no ids; and the same with ids (the key pass writes them)."""
    n = 1 << 28
    cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(3)]
    for c, seed in zip(cols, (2, 102, 103)):
        ragen.int32_column_dev(seed, c)
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    hc = [c.cpu().numpy() for c in cols]
    exp_ids, exp = oracle.select_rows(hc[0], preds, [hc[0], hc[1], hc[2]])
    for rowids in (False, True):
        ids, outs, cnt = R.select_rows(cols[0], preds, [cols[0], cols[1], cols[2]], rowids=rowids)
        torch.cuda.synchronize()
        c = int(cnt.item())
        assert c == exp_ids.size
        if rowids:
            np.testing.assert_array_equal(ids[:c].cpu().numpy().astype(np.int64), exp_ids)
        for o, e in zip(outs, exp):
            np.testing.assert_array_equal(o[:c].cpu().numpy(), e)



def test_row_ids_near_2_pow_32(R):
    """n = 2^32 - 5 rows (the ABI limit for uint32 ids): key[i] = int32(i)
    (wrapping), select key < 0 keeps rows 2^31 .. n-1, so ids run up to
    2^32 - 6 and each output is known in closed form; with ids (key pass) and
    without (dense compaction path), sampled positions checked."""
    n = (1 << 32) - 5
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    step = 1 << 28
    for lo in range(0, n, step):
        hi = min(n, lo + step)
        x[lo:hi].copy_(torch.arange(lo, hi, dtype=torch.int64, device="cuda").to(torch.int32))
    c_exp = n - (1 << 31)
    rng = np.random.default_rng(1)
    pos = np.concatenate([np.arange(64), rng.integers(0, c_exp, 1 << 16), np.arange(c_exp - 64, c_exp)])
    pd = torch.from_numpy(pos).cuda()
    for rowids in (True, False):
        ids, outs, cnt = R.select_rows(x, [("lt", 0)], [x], rowids=rowids)
        torch.cuda.synchronize()
        assert int(cnt.item()) == c_exp
        exp_rows = (1 << 31) + pos
        if rowids:
            np.testing.assert_array_equal(ids.view(torch.int32)[pd].cpu().numpy().view(np.uint32).astype(np.int64),
                                          exp_rows)
        np.testing.assert_array_equal(outs[0][pd].cpu().numpy().astype(np.int64), exp_rows - (1 << 32))
        del ids, outs
