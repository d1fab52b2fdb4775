"""GPU parity: libra.so's fused / unfused SELECT chain vs the CPU oracle.

Bit-exact comparison of the selected values (order-preserving, unique result)
and of the count, on seeded inputs from ragen; sizes span several 4096-row
tiles, ragged tails, misaligned starts, and BASELINE's 2^20 / 2^28 configs.
"""
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


def run(R, x_np, preds, fused=True, offset=0, out_cap=None):
    xt = torch.from_numpy(np.concatenate([np.zeros(offset, np.int32), x_np])).cuda()
    x = xt[offset:]
    out = None
    if out_cap is not None:
        out = torch.full((max(1, out_cap),), -7, dtype=torch.int32, device="cuda")
    o, c = R.select_chain(x, preds, fused=fused, out=out)
    torch.cuda.synchronize()
    c = int(c.item())
    return o.cpu().numpy(), c


SIZES = [0, 1, 3, 4, 5, 4095, 4096, 4097, 8191, 12289, 100003, 1 << 20]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("offset", [0, 1, 3])
def test_single_select_sizes_and_alignment(R, n, offset):
    x = ragen.int32_column(100 + n, n)
    preds = [("lt", 0)]
    exp = oracle.select(x, preds)
    got, c = run(R, x, preds, offset=offset)
    assert c == exp.size
    np.testing.assert_array_equal(got[:c], exp)


@pytest.mark.parametrize("s", [0.01, 0.1, 0.25, 0.5, 0.75, 0.9])
@pytest.mark.parametrize("k", [1, 2, 3])
@pytest.mark.parametrize("fused", [True, False])
def test_nested_chain_selectivity_sweep(R, s, k, fused):
    n = (1 << 20) + 777
    x = ragen.int32_column(2, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(s, k)]
    exp = oracle.select(x, preds)
    got, c = run(R, x, preds, fused=fused)
    assert c == exp.size
    np.testing.assert_array_equal(got[:c], exp)


OPS = ["lt", "le", "gt", "ge", "eq", "ne"]


@settings(max_examples=60, deadline=None)
@given(preds=st.lists(st.tuples(st.sampled_from(OPS), st.integers(-6, 6)), max_size=8),
       n=st.integers(0, 20000), seed=st.integers(0, 1000), fused=st.booleans())
def test_random_chains_small_domain(R, preds, n, seed, fused):
    """Values in [-8, 8] so EQ/NE and range folding all matter."""
    rng = np.random.default_rng(seed)
    x = rng.integers(-8, 9, n).astype(np.int32)
    exp = oracle.select(x, preds)
    got, c = run(R, x, preds, fused=fused, offset=seed % 4)
    assert c == exp.size
    np.testing.assert_array_equal(got[:c], exp)


@pytest.mark.parametrize("preds", [
    [("lt", -(2**31))], [("gt", 2**31 - 1)], [("ge", -(2**31))], [("le", 2**31 - 1)], [],
    [("eq", -(2**31))], [("ne", 2**31 - 1), ("ne", -(2**31))], [("gt", 5), ("lt", 5)],
    [("ge", 0), ("le", 0), ("ne", 0)], [("gt", -(10**9)), ("lt", 10**9), ("ne", 3), ("ne", 4)],
])
def test_extreme_predicates(R, preds):
    x = ragen.int32_column(9, 50000)
    x[:6] = [-(2**31), 2**31 - 1, 0, 3, 4, 5]
    exp = oracle.select(x, preds)
    for fused in (True, False):
        got, c = run(R, x, preds, fused=fused)
        assert c == exp.size
        np.testing.assert_array_equal(got[:c], exp)


@pytest.mark.parametrize("lg", [23, 25])
@pytest.mark.parametrize("s,k", [(0.01, 1), (0.1, 1), (0.5, 2), (0.6, 1), (0.75, 1), (0.9, 1), (1.0, 0)])
def test_many_tiles_per_cta(R, lg, s, k):
    """Several 8192-row tiles per CTA: exercises the ring of selected rows
    (contiguous runs, wrap-around, early writes when it runs short) and the
    lagged / on-demand look-back."""
    n = (1 << lg) + 12345
    x = ragen.int32_column(60 + lg, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(s, k)]
    exp = oracle.select(x, preds)
    got, c = run(R, x, preds)
    assert c == exp.size
    np.testing.assert_array_equal(got[:c], exp)


def test_selectivity_zero_one_identity(R):
    x = ragen.int32_column(4, 300001)
    got, c = run(R, x, [("lt", -(2**31))])
    assert c == 0
    got, c = run(R, x, [])
    assert c == x.size
    np.testing.assert_array_equal(got[:c], x)


def test_out_cap_truncates_but_counts(R):
    x = ragen.int32_column(5, 100000)
    preds = [("lt", 0)]
    exp = oracle.select(x, preds)
    got, c = run(R, x, preds, out_cap=1000)
    assert c == exp.size
    np.testing.assert_array_equal(got[:1000], exp[:1000])


def test_workspace_reuse_across_sizes(R):
    """Self-cleaning status words: successive calls with varying n on one workspace."""
    for i, n in enumerate([1 << 20, 5, 0, 70000, 1 << 18, 1, (1 << 20) + 3, 4096, 0, 123457]):
        x = ragen.int32_column(1000 + i, n)
        preds = [("ge", -(2**30)), ("lt", 2**29)]
        exp = oracle.select(x, preds)
        got, c = run(R, x, preds)
        assert c == exp.size, (i, n)
        np.testing.assert_array_equal(got[:c], exp)


def test_many_back_to_back_calls_same_stream(R):
    n = 1 << 16
    x = torch.from_numpy(ragen.int32_column(77, n)).cuda()
    preds = [("lt", 0)]
    exp = oracle.select(x.cpu().numpy(), preds)
    outs = [R.select_chain(x, preds) for _ in range(50)]
    torch.cuda.synchronize()
    for o, c in outs:
        assert int(c.item()) == exp.size
        np.testing.assert_array_equal(o[: exp.size].cpu().numpy(), exp)


def test_full_size_config_2_pow_28(R):
    """BASELINE configs[1] at its full size, in the launch configuration bench.py
    times (device-generated column, k=2, s=0.5): full comparison vs the oracle."""
    n = 1 << 28
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(2, x)
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    out, c = R.select_chain(x, preds)
    torch.cuda.synchronize()
    c = int(c.item())
    xh = x.cpu().numpy()
    np.testing.assert_array_equal(xh, ragen.int32_column(2, n))  # device gen == host gen
    exp = oracle.select(xh, preds)
    assert c == exp.size
    np.testing.assert_array_equal(out[:c].cpu().numpy(), exp)
    out2, c2 = R.select_chain(x, preds, fused=False)
    torch.cuda.synchronize()
    assert int(c2.item()) == c
    assert torch.equal(out2[:c], out[:c])


def test_bad_arguments_raise(R):
    x = torch.zeros(10, dtype=torch.int32, device="cuda")
    with pytest.raises(R.RAError) as e:
        R.select_chain(x, [(9, 0)])
    assert e.value.code == R.RA_E_INVAL
    with pytest.raises(R.RAError):
        R.select_chain(x, [("lt", 0)] * 9)


def test_more_than_2_pow_31_rows(R):
    """2^31 + 2^28 + 12345 rows (9.7 GB in, > 2^18 tiles, output offsets past
    2^31): 64-bit tile indices, tickets and offsets; count and sampled outputs
    vs the oracle's definition evaluated with numpy on the same rows."""
    n = (1 << 31) + (1 << 28) + 12345
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(12, x)
    preds = [("gt", -(2**31) + 2**28)]  # keeps ~94%: the output passes 2^31 rows
    out, c = R.select_chain(x, preds)
    torch.cuda.synchronize()
    c = int(c.item())
    xh = x.cpu().numpy()
    keep = xh > -(2**31) + 2**28
    assert c == int(keep.sum()), (c, int(keep.sum()))
    assert c > (1 << 31)
    idx = np.flatnonzero(keep)
    rng = np.random.default_rng(0)
    pos = np.concatenate([np.arange(64), rng.integers(0, c, 1 << 16), np.arange(c - 64, c)])
    np.testing.assert_array_equal(out[torch.from_numpy(pos).cuda()].cpu().numpy(), xh[idx[pos]])


@pytest.mark.parametrize("extra", [1, 4, 8, 255, 4096 + 3])
def test_unfused_workspace_larger_than_required(R, extra):
    """ws_bytes may exceed the required size by any amount (ra.h): the unfused
    intermediates are placed from the 256-B aligned end, so an odd or
    non-multiple-of-8 ws_bytes cannot misalign them."""
    n = 100_003
    x = torch.from_numpy(ragen.int32_column(55, n)).cuda()
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 3)]
    exp = oracle.select(x.cpu().numpy(), preds)
    need = R.ra_select_workspace_bytes(n, 3, 0)
    ws = torch.zeros(need + extra + 256, dtype=torch.uint8, device="cuda")
    out = torch.empty(n, dtype=torch.int32, device="cuda")
    cnt = torch.empty(1, dtype=torch.int64, device="cuda")
    P = R.make_preds(preds)
    R.ra_select_chain(x.data_ptr(), n, P, 3, 0, out.data_ptr(), n, cnt.data_ptr(), ws.data_ptr(), need + extra,
                      int(torch.cuda.current_stream().cuda_stream))
    torch.cuda.synchronize()
    assert int(cnt.item()) == exp.size
    np.testing.assert_array_equal(out[:exp.size].cpu().numpy(), exp)


@pytest.mark.parametrize("base", [0, 1 << 21], ids=["single_output_kernel", "multi_output_pass"])
def test_epoch_tag_wrap_clears_stale_status_words(R, base):
    """Status words carry a 28-bit launch tag.  A word left by a launch exactly
    2^28 launches earlier carries the tag the wrapped epoch will use again: the
    launch before the wrap must clear every word the workspace has held (header
    high-water mark), so a later, larger launch never reads such a word as a
    published aggregate.  Simulated by planting the header and stale words."""
    n_small, n_big = base + 5 * 8192 + 11, base + 40 * 8192 + 5
    hw = (n_big + 8191) // 8192 + 7  # words carried so far: more than the big launch's tiles
    ws = torch.zeros(R.ra_select_workspace_bytes(n_big, 1, 1), dtype=torch.uint8, device="cuda")
    words = ws[256:].view(torch.int64)
    hdr32, hdr64 = ws[:256].view(torch.int32), ws[:256].view(torch.int64)
    flag_a, tag_shift = 1 << 62, 34
    # stale words of "tag 0" (a launch 2^28 launches ago) with bogus aggregates
    words[:hw] = flag_a | (0 << tag_shift) | 1000
    hdr32[0] = (1 << 28) - 1      # this launch uses the last tag before the wrap
    hdr64[3] = hw                 # high-water mark: hw words carried so far
    preds = [("lt", 0)]
    sh = int(torch.cuda.current_stream().cuda_stream)
    P = R.make_preds(preds)
    for n in (n_small, n_big, n_big):  # tags 2^28-1, then 0 (the wrap), then 1
        x = torch.from_numpy(ragen.int32_column(n, n)).cuda()
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        cnt = torch.empty(1, dtype=torch.int64, device="cuda")
        R.ra_select_chain(x.data_ptr(), n, P, 1, 1, out.data_ptr(), n, cnt.data_ptr(), ws.data_ptr(), ws.numel(), sh)
        torch.cuda.synchronize()
        exp = oracle.select(x.cpu().numpy(), preds)
        assert int(cnt.item()) == exp.size, n
        np.testing.assert_array_equal(out[:exp.size].cpu().numpy(), exp)
    assert int(hdr32[0].item()) == (1 << 28) + 2 and int(hdr64[3].item()) == hw


@pytest.mark.parametrize("big", [False, True])
def test_epoch_advances_once_per_launch_even_without_tiles(R, big):
    """The epoch is advanced by the last CTA out (so every CTA of a launch,
    also one that drew no tile, uses the same tag), once per launch — also for
    n = 0.  A wrap that falls on an empty launch still clears the stale words:
    planted "tag 0" words must not read as published in the next launch.
    big: above 2^21 rows (multi-output pass), else the single-output pass."""
    n_big = (1 << 21) + 40 * 8192 + 5 if big else 40 * 8192 + 5
    ws = torch.zeros(R.ra_select_workspace_bytes(n_big, 1, 1), dtype=torch.uint8, device="cuda")
    hw = min((n_big + 8191) // 8192 + 7, (ws.numel() - 256) // 8)  # >= the big launch's tiles
    words = ws[256:].view(torch.int64)
    hdr32, hdr64 = ws[:256].view(torch.int32), ws[:256].view(torch.int64)
    words[:hw] = (1 << 62) | 1000          # stale "tag 0" words with bogus aggregates
    hdr32[0] = (1 << 28) - 1               # the next launch is the last before the wrap
    hdr64[3] = hw
    preds = [("lt", 0)]
    sh = int(torch.cuda.current_stream().cuda_stream)
    P = R.make_preds(preds)
    empty = torch.empty(1, dtype=torch.int32, device="cuda")
    cnt = torch.full((1,), -1, dtype=torch.int64, device="cuda")
    R.ra_select_chain(empty.data_ptr(), 0, P, 1, 1, empty.data_ptr(), 0, cnt.data_ptr(), ws.data_ptr(), ws.numel(), sh)
    torch.cuda.synchronize()
    assert int(cnt.item()) == 0 and int(hdr32[0].item()) == 1 << 28
    x = torch.from_numpy(ragen.int32_column(7, n_big)).cuda()
    out = torch.empty(n_big, dtype=torch.int32, device="cuda")
    R.ra_select_chain(x.data_ptr(), n_big, P, 1, 1, out.data_ptr(), n_big, cnt.data_ptr(), ws.data_ptr(), ws.numel(), sh)
    torch.cuda.synchronize()
    exp = oracle.select(x.cpu().numpy(), preds)
    assert int(cnt.item()) == exp.size
    np.testing.assert_array_equal(out[:exp.size].cpu().numpy(), exp)
    assert int(hdr32[0].item()) == (1 << 28) + 1


def test_select_rows_workspace_reuse_across_sizes(R):
    """Tuple SELECT keeps its order masks and staged ids at the END of the
    workspace: a later call with larger n on the same (bigger) workspace never
    reads an earlier call's masks as tile status words."""
    big = 3 << 20
    R.select_rows(torch.zeros(big, dtype=torch.int32, device="cuda"), [("lt", 0)])
    for i, n in enumerate([1 << 16, (1 << 20) + 3, 5000, 1 << 21]):
        key = ragen.int32_column(300 + i, n)
        pay = ragen.int32_column(400 + i, n)
        preds = [("lt", -(2**31) + 2**26)]  # ~1.6%: sparse masks (isolated bits)
        exp_ids = np.flatnonzero(key < -(2**31) + 2**26)
        ids, outs, cnt = R.select_rows(torch.from_numpy(key).cuda(), preds, [torch.from_numpy(pay).cuda()])
        torch.cuda.synchronize()
        c = int(cnt.item())
        assert c == exp_ids.size
        np.testing.assert_array_equal(ids[:c].cpu().numpy().astype(np.int64), exp_ids)
        np.testing.assert_array_equal(outs[0][:c].cpu().numpy(), pay[exp_ids])


def test_one_workspace_across_both_pass_kinds(R):
    """The fused chain runs the single-output kernel up to 2^21 rows and the
    multi-output pass above (same header, same one-word-per-8192-row status
    format): one workspace alternating between them, sizes on both sides of
    the threshold, every result exact."""
    sizes = [(1 << 21) - 7, (1 << 21) + 9, 1 << 20, 3 << 21, 12345, (1 << 22) + 1, 1 << 21, 5, (1 << 21) + 1]
    ws_b = R.ra_select_workspace_bytes(max(sizes), 2, 1)
    ws = torch.zeros(ws_b, dtype=torch.uint8, device="cuda")
    sh = int(torch.cuda.current_stream().cuda_stream)
    for i, n in enumerate(sizes):
        x = torch.from_numpy(ragen.int32_column(500 + i, n)).cuda()
        preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        cnt = torch.empty(1, dtype=torch.int64, device="cuda")
        R.ra_select_chain(x.data_ptr(), n, R.make_preds(preds), 2, 1, out.data_ptr(), n, cnt.data_ptr(),
                          ws.data_ptr(), ws_b, sh)
        torch.cuda.synchronize()
        exp = oracle.select(x.cpu().numpy(), preds)
        assert int(cnt.item()) == exp.size, (i, n)
        np.testing.assert_array_equal(out[:exp.size].cpu().numpy(), exp)


@pytest.mark.parametrize("s", [0.01, 0.25, 0.5, 0.9])
@pytest.mark.parametrize("k", [1, 3])
def test_chain_sweep_multi_output_pass(R, s, k):
    """The selectivity sweep above 2^21 rows (the fused chain's warp-specialised
    pass), with a misaligned start and a ragged tail."""
    n = (1 << 22) + 777
    x = ragen.int32_column(3, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(s, k)]
    exp = oracle.select(x, preds)
    got, c = run(R, x, preds, offset=1)
    assert c == exp.size
    np.testing.assert_array_equal(got[:c], exp)
