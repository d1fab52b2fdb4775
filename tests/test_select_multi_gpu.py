"""GPU parity of several SELECTs on one input (ra_select_multi, SURVEY §8(f)
f2, Fig 2(c)) through the C-ABI against the CPU oracle (oracle.select_multi):
each output bit-exact and in input order, over ragged/misaligned inputs, many
tiles, every selectivity regime, != predicates, capacity limits, and
interleaved with single-output calls on the same workspace."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
import ragen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def R():
    import paper_conf_ipps_wudwcyc12_b200 as R
    return R


def check(R, x, chains, offset=0):
    xd = torch.from_numpy(np.concatenate([np.zeros(offset, np.int32), x])).cuda()[offset:]
    outs, cnt = R.select_multi(xd, chains)
    torch.cuda.synchronize()
    exp = oracle.select_multi(x, chains)
    for o, (out, e) in enumerate(zip(outs, exp)):
        c = int(cnt[o].item())
        assert c == e.size, (o, c, e.size)
        assert np.array_equal(out[:c].cpu().numpy(), e), o


@pytest.mark.parametrize("n", [0, 1, 5, 8191, 8192, 8193, 5 * 8192 + 1234, 1_000_003])
@pytest.mark.parametrize("offset", [0, 1, 2, 3])
def test_sizes_offsets(R, n, offset):
    x = ragen.int32_column(71 + n, n)
    check(R, x, [[("lt", 0)], [("gt", -(2**29)), ("lt", 2**30)]], offset)
    check(R, x, [[("gt", -(2**31) + 2**28)], [("ne", 7)]], offset)  # both dense


@pytest.mark.parametrize("s0,s1", [(0.0, 1.0), (0.01, 0.9), (0.5, 0.5), (0.9, 0.9), (1.0, 1.0), (0.25, 0.75)])
def test_selectivities_many_tiles(R, s0, s1):
    n = (1 << 22) + 333
    x = ragen.int32_column(72, n)

    def chain(s):
        if s == 0.0:
            return [("lt", -(2**31))]
        if s == 1.0:
            return [("ge", -(2**31))]
        return [("lt", ragen.nested_thresholds(s, 1)[0])]
    check(R, x, [chain(s0), chain(s1)])


def test_complementary_and_ne(R):
    n = 2_000_001
    x = ragen.int32_column(73, n)
    t = int(x[999])
    check(R, x, [[("lt", t)], [("ge", t)]])
    check(R, x, [[("ne", int(x[5])), ("ne", int(x[6])), ("lt", 2**30)], [("eq", int(x[7]))]])
    check(R, x, [[], [("le", 0)]])  # k = 0: identity output


def test_single_output_and_shared_workspace(R):
    n = 300_007
    x = ragen.int32_column(74, n)
    xd = torch.from_numpy(x).cuda()
    check(R, x, [[("lt", 12345)]])
    for _ in range(3):  # alternate single-output and dual-output launches on one workspace
        out, c = R.select_chain(xd, [("gt", 0)])
        outs, cnt = R.select_multi(xd, [[("lt", 0)], [("gt", 0)]])
        torch.cuda.synchronize()
        e = x[x > 0]
        assert int(c.item()) == e.size and np.array_equal(out[:e.size].cpu().numpy(), e)
        assert np.array_equal(outs[1][:int(cnt[1].item())].cpu().numpy(), e)


def test_capacity(R):
    n = 400_000
    x = ragen.int32_column(75, n)
    xd = torch.from_numpy(x).cuda()
    outs = [torch.empty(1000, dtype=torch.int32, device="cuda"), torch.empty(n, dtype=torch.int32, device="cuda")]
    outs, cnt = R.select_multi(xd, [[("lt", 0)], [("gt", 0)]], outs=outs)
    torch.cuda.synchronize()
    e0, e1 = x[x < 0], x[x > 0]
    assert int(cnt[0].item()) == e0.size and int(cnt[1].item()) == e1.size
    assert np.array_equal(outs[0].cpu().numpy(), e0[:1000])
    assert np.array_equal(outs[1][:e1.size].cpu().numpy(), e1)


@pytest.mark.parametrize("caps", [(1000, 5), (3 * 8192 + 17, 10**9), (0, 123457)])
def test_capacity_dense_outputs(R, caps):
    """Both outputs keep ~90% of every tile, more than the selected-row ring
    holds at once: compaction waits for the writers; truncation stays exact
    and nothing is written past either capacity."""
    n = 50 * 8192 + 99
    x = ragen.int32_column(76, n)
    xd = torch.from_numpy(x).cuda()
    chains = [[("lt", ragen.nested_thresholds(0.9, 1)[0])], [("gt", -ragen.nested_thresholds(0.9, 1)[0])]]
    e0, e1 = oracle.select_multi(x, chains)
    cap = [min(c, n) for c in caps]
    outs = [torch.full((c + 64,), -3, dtype=torch.int32, device="cuda") for c in cap]
    P = [R.make_preds(c) for c in chains]
    import ctypes
    mch = (ctypes.c_void_p * 2)(*[ctypes.addressof(p_) for p_ in P])
    mks = (ctypes.c_int * 2)(1, 1)
    mop = (ctypes.c_void_p * 2)(*[o.data_ptr() for o in outs])
    mcap = (ctypes.c_int64 * 2)(*cap)
    cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
    mcp = (ctypes.c_void_p * 2)(cnt.data_ptr(), cnt.data_ptr() + 8)
    wsb = R.ra_select_multi_workspace_bytes(n)
    ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
    R.ra_select_multi(xd.data_ptr(), n, mch, mks, 2, mop, mcap, mcp, ws.data_ptr(), wsb, 0)
    torch.cuda.synchronize()
    assert [int(v) for v in cnt.cpu().tolist()] == [e0.size, e1.size]
    for o, e, c in zip(outs, (e0, e1), cap):
        h = o.cpu().numpy()
        m = min(c, e.size)
        assert np.array_equal(h[:m], e[:m])
        assert (h[m:] == -3).all()


def test_argument_errors(R):
    xd = torch.zeros(16, dtype=torch.int32, device="cuda")
    with pytest.raises(R.RAError) as e:
        R.select_multi(xd, [[("lt", 0)]] * (R.RA_MAX_OUTPUTS + 1))
    assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError) as e:
        R.select_multi(xd, [[("lt", 0)], [(7, 0)]])
    assert e.value.code == R.RA_E_INVAL


def _chain(s):
    if s == 0.0:
        return [("lt", -(2**31))]
    if s == 1.0:
        return [("ge", -(2**31))]
    return [("lt", ragen.nested_thresholds(s, 1)[0])]


@pytest.mark.parametrize("n", [0, 1, 5, 4095, 4096, 4097, 7 * 4096 + 1234, 1_000_003])
@pytest.mark.parametrize("offset", [0, 3])
@pytest.mark.parametrize("M", [3, 4])
def test_three_four_outputs_sizes_offsets(R, n, offset, M):
    x = ragen.int32_column(171 + n, n)
    chains = [[("lt", 0)], [("gt", -(2**29)), ("lt", 2**30)], [("ne", int(x[0]) if n else 3)], [("ge", 2**30)]][:M]
    check(R, x, chains, offset)


@pytest.mark.parametrize("sel", [(0.0, 0.0, 0.0, 0.0), (1.0, 1.0, 1.0, 1.0), (0.9, 0.9, 0.9, 0.9),
                                 (0.01, 0.5, 0.99, 0.25), (0.5, 0.5, 0.5), (1.0, 0.0, 1.0), (0.9, 0.9)])
def test_many_outputs_selectivities_many_tiles(R, sel):
    """Up to four outputs, every one dense (a tile's M runs fill most of the
    ring), empty, or mixed; 2^22+ rows = hundreds of tiles per SM."""
    n = (1 << 22) + 333
    x = ragen.int32_column(172, n)
    check(R, x, [_chain(s) for s in sel])


@settings(max_examples=40, deadline=None)
@given(st.integers(1, 4), st.integers(0, 70000), st.integers(0, 3), st.data())
def test_random_chains_brute_force(R, M, n, offset, data):
    """Random predicate chains (all six ops, up to 8 per output) on random
    data; each output vs the oracle (itself pinned by brute force)."""
    rng = np.random.default_rng(n * 7 + M)
    x = rng.integers(-50, 50, n, dtype=np.int32) if n % 2 else rng.integers(-(2**31), 2**31, n, dtype=np.int64).astype(np.int32)
    ops = ["lt", "le", "gt", "ge", "eq", "ne"]
    chains = []
    for _ in range(M):
        k = data.draw(st.integers(0, 8))
        chains.append([(data.draw(st.sampled_from(ops)), data.draw(st.integers(-60, 60))) for _ in range(k)])
    check(R, x, chains, offset)


def test_workspace_shared_across_output_counts(R):
    """One workspace, successive launches with M = 1..4 (tile size 8192 for
    M <= 2, 4096 for M >= 3: different status-word layouts on the same words)."""
    n = 3 * (1 << 20) + 11
    x = ragen.int32_column(174, n)
    xd = torch.from_numpy(x).cuda()
    chains = [[("lt", 0)], [("gt", -(2**30))], [("ne", 5), ("lt", 2**30)], [("ge", -(2**29))]]
    exp = oracle.select_multi(x, chains)
    for M in (4, 1, 3, 2, 4, 4, 1, 2, 3):
        outs, cnt = R.select_multi(xd, chains[:M])
        torch.cuda.synchronize()
        for o in range(M):
            c = int(cnt[o].item())
            assert c == exp[o].size, (M, o)
            assert np.array_equal(outs[o][:c].cpu().numpy(), exp[o]), (M, o)


def test_full_size_four_outputs(R):
    """2^28 device-generated rows (seed 2), four outputs (.5, .5, .25, .25):
    the bench's M = 4 shape, full comparison with the oracle."""
    n = 1 << 28
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(2, x)
    chains = [[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)], [("ge", 2**30)], [("lt", -(2**30))]]
    outs, cnt = R.select_multi(x, chains)
    torch.cuda.synchronize()
    exp = oracle.select_multi(x.cpu().numpy(), chains)
    for o, c, e in zip(outs, cnt.cpu().tolist(), exp):
        assert int(c) == e.size
        np.testing.assert_array_equal(o[:int(c)].cpu().numpy(), e)


@pytest.mark.parametrize("pair", ["identical", "nested", "complementary"])
def test_two_outputs_ring_pressure(R, pair):
    """Two outputs keeping ~half (or all) of 2^24 rows each with overlapping
    predicates: the regime where the ring of selected rows runs full (2 input
    slots for M = 2, placements on demand), and the two outputs' offsets move
    in lockstep.  Full comparison with the oracle, 4 launches on one workspace."""
    n = 1 << 24
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(11, x)
    chains = {"identical": [[("lt", 0)], [("lt", 0)]],
              "nested": [[("lt", 2**30)], [("ge", -(2**31))]],
              "complementary": [[("lt", 0)], [("ge", 0)]]}[pair]
    exp = oracle.select_multi(x.cpu().numpy(), chains)
    outs = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(2)]
    for _ in range(4):
        _, cnt = R.select_multi(x, chains, outs=outs)
        torch.cuda.synchronize()
        for o, c, e in zip(outs, cnt.cpu().tolist(), exp):
            assert int(c) == e.size
            np.testing.assert_array_equal(o[:int(c)].cpu().numpy(), e)


def test_full_size_bench_config(R):
    """bench.py's f2 leg at full size (2^28 device-generated rows, seed 2, the
    bench's two chains), full comparison of both outputs with the oracle."""
    n = 1 << 28
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(2, x)
    chains = [[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)]]
    outs, cnt = R.select_multi(x, chains)
    torch.cuda.synchronize()
    exp = oracle.select_multi(x.cpu().numpy(), chains)
    for o, c, e in zip(outs, cnt.cpu().tolist(), exp):
        assert int(c) == e.size
        np.testing.assert_array_equal(o[:int(c)].cpu().numpy(), e)



@pytest.mark.parametrize("M", [2, 4])
def test_outputs_past_2_pow_31_rows_closed_form(R, M):
    """n = 2^31 + 2^28 rows with key[i] = int32(i) (wrapping).  Outputs:
    key >= 0 (rows 0 .. 2^31-1: 2^31 outputs, the last at position 2^31 - 1),
    key < 2^30 (rows 0 .. 2^30-1, then the wrapped rows 2^31 .. n-1),
    key < 0 (the wrapped rows), key >= 2^30 (rows 2^30 .. 2^31-1).  Counts
    exact (64-bit offsets past 2^31), sampled outputs against the closed form."""
    n = (1 << 31) + (1 << 28)
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    step = 1 << 28
    for lo in range(0, n, step):
        x[lo:lo + step].copy_(torch.arange(lo, lo + step, dtype=torch.int64, device="cuda").to(torch.int32))
    chains = [[("ge", 0)], [("lt", 1 << 30)], [("lt", 0)], [("ge", 1 << 30)]][:M]
    outs, cnt = R.select_multi(x, chains)
    torch.cuda.synchronize()
    del x
    cs = [int(v) for v in cnt.cpu().tolist()][:M]
    exp_counts = [1 << 31, (1 << 30) + (1 << 28), 1 << 28, 1 << 30][:M]
    assert cs == exp_counts
    closed = [lambda p: p,
              lambda p: np.where(p < (1 << 30), p, p - (1 << 30) + (1 << 31) - (1 << 32)),
              lambda p: p - (1 << 31),
              lambda p: p + (1 << 30)]
    rng = np.random.default_rng(2)
    for o in range(M):
        c = cs[o]
        pos = np.concatenate([np.arange(64), rng.integers(0, c, 1 << 16), np.arange(c - 64, c)])
        got = outs[o][torch.from_numpy(pos).cuda()].cpu().numpy().astype(np.int64)
        np.testing.assert_array_equal(got, closed[o](pos))
