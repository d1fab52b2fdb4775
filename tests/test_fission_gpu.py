"""GPU parity: ra_fission_run (host-resident chain, chunked over streams) vs
the oracle; fission == device-resident == oracle for every chunk/stream mix."""
import numpy as np
import pytest

import oracle
import ragen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def R():
    import paper_conf_ipps_wudwcyc12_b200 as R
    return R


@pytest.fixture(scope="module")
def streams():
    return [torch.cuda.Stream() for _ in range(4)]


def pinned(a):
    t = torch.empty(a.size, dtype=torch.int32, pin_memory=True)
    t.numpy()[:] = a
    return t


@pytest.mark.parametrize("n", [0, 1, 4097, 1_000_003])
@pytest.mark.parametrize("chunk", [1 << 12, 100_000, 1 << 20, 1 << 30])
@pytest.mark.parametrize("nstreams", [1, 2, 3, 4])
def test_fission_matches_oracle(R, streams, n, chunk, nstreams):
    if n > 100_000 and chunk == 1 << 12 and nstreams != 3:
        pytest.skip("covered by the 3-stream case")
    x = ragen.int32_column(40 + n, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    exp = oracle.select(x, preds)
    h_out, c = R.fission_run(pinned(x), preds, chunk, streams[:nstreams])
    assert c == exp.size
    np.testing.assert_array_equal(h_out.numpy()[:c], exp)


@pytest.mark.parametrize("fused", [True, False])
@pytest.mark.parametrize("k", [0, 1, 3])
def test_fission_modes(R, streams, fused, k):
    n = 3_000_001
    x = ragen.int32_column(41, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(0.7, k)]
    exp = oracle.select_chunked(x, preds, 1 << 20)
    h_out, c = R.fission_run(pinned(x), preds, 1 << 20, streams[:3], fused=fused)
    assert c == exp.size
    np.testing.assert_array_equal(h_out.numpy()[:c], exp)


def test_fission_capacity(R, streams):
    x = ragen.int32_column(42, 200000)
    preds = [("lt", 0)]
    exp = oracle.select(x, preds)
    h_out = torch.empty(1000, dtype=torch.int32, pin_memory=True)
    _, c = R.fission_run(pinned(x), preds, 50000, streams[:2], h_out=h_out)
    assert c == exp.size
    np.testing.assert_array_equal(h_out.numpy(), exp[:1000])


def test_fission_requires_pinned(R, streams):
    import ctypes
    x = np.arange(1000, dtype=np.int32)
    out = np.empty(1000, dtype=np.int32)
    counts = np.zeros(1, dtype=np.int64)
    P = R.make_preds([("lt", 0)])
    sarr = (ctypes.c_void_p * 1)(streams[0].cuda_stream)
    ws = torch.zeros(R.ra_fission_workspace_bytes(1000, 1, 1, 1), dtype=torch.uint8, device="cuda")
    cnt = ctypes.c_int64()
    with pytest.raises(R.RAError) as e:
        R.ra_fission_run(x.ctypes.data, 1000, P, 1, 1, 1000, sarr, 1, out.ctypes.data, 1000,
                         ctypes.byref(cnt), counts.ctypes.data, ws.data_ptr(), ws.numel())
    assert e.value.code == R.RA_E_NOT_PINNED


def test_full_size_config_3_host_resident_2_pow_30(R, streams):
    """BASELINE configs[3] at full size, in bench.py's launch configuration:
    2^30 host-resident rows (seed 4) in pinned memory, k=2 s=.5/stage, chunk
    2^24, 3 streams; full comparison with the oracle (chunked SELECT equals
    SELECT, pinned in test_oracle_select)."""
    n = 1 << 30
    h = torch.empty(n, dtype=torch.int32, pin_memory=True)
    ragen.int32_column(4, n, out=h.numpy())
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    h_out, c = R.fission_run(h, preds, 1 << 24, streams[:3])
    exp = oracle.select(h.numpy(), preds)
    assert c == exp.size
    np.testing.assert_array_equal(h_out.numpy()[:c], exp)


@pytest.mark.parametrize("chunk", [(1 << 22) + 5, (1 << 21) + 1, 3 << 20])
@pytest.mark.parametrize("nstreams", [1, 3])
def test_fission_chunks_above_the_small_pass_threshold(R, streams, chunk, nstreams):
    """Chunks above 2^21 rows run the multi-output pass per chunk, smaller
    trailing chunks the single-output kernel: ragged chunking over 5M rows,
    equal to the oracle."""
    n = 5_000_003
    x = ragen.int32_column(90, n)
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    exp = oracle.select(x, preds)
    h_out, c = R.fission_run(pinned(x), preds, chunk, streams[:nstreams])
    assert c == exp.size
    assert np.array_equal(h_out[:c].numpy(), exp)
