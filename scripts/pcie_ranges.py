"""PCIe evidence for the fission paths: one call of each, bench-sized, inside a
cudaProfilerStart/Stop range, for ncu's application-range replay:

  ncu --replay-mode app-range --profile-from-start off \
      --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,gpu__time_duration.sum \
      --csv --log-file gpurun_out/pcie.csv python scripts/pcie_ranges.py

Ranges, in order (names printed to stdout, one per line):
  select_fission_n28    ra_fission_run, 2^28 int32 rows (seed 2), k=2 s=.5, chunk 2^24, 3 streams  (bench e2e)
  select_fission_n30    ra_fission_run, 2^30 rows (seed 4), same chain and chunking                (configs[3])
  q1_fission_sf10       ra_q1_fission_run, SF10 wide, chunk 2^22, 3 streams                       (q1_sf10.e2e)
  q1n_fission_sf10      ra_q1_narrow_fission_run, SF10 narrow, chunk 2^23, 3 streams              (q1_sf10.e2e.narrow)
Outside ncu it also times each call (CUDA events) and prints the H2D GB/s.
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
import ragen  # noqa: E402


def ranged(name, fn, h2d_bytes):
    fn()  # warm-up (workspace, first-call costs) outside the range
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    t0 = time.perf_counter()
    fn()
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    torch.cuda.profiler.stop()
    print(f"{name} {dt * 1e3:.2f} ms host wall, H2D {h2d_bytes / dt / 1e9:.1f} GB/s ({h2d_bytes} bytes)", flush=True)


def main():
    torch.cuda.set_device(0)
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    st = [torch.cuda.Stream() for _ in range(3)]
    for name, seed, lg in (("select_fission_n28", 2, 28), ("select_fission_n30", 4, 30)):
        n = 1 << lg
        h = torch.empty(n, dtype=torch.int32, pin_memory=True)
        ragen.int32_column(seed, n, out=h.numpy())
        o = torch.empty(n, dtype=torch.int32, pin_memory=True)
        cc = torch.zeros(n >> 24, dtype=torch.int64, pin_memory=True)
        ranged(name, lambda: R.fission_run(h, preds, 1 << 24, st, h_out=o, h_chunk_counts=cc), 4 * n)
        del h, o
    N = ragen.rows_for_sf(10)
    cols = ragen.lineitem(5, N, ragen.parts_for_sf(10))
    hw = {k: torch.from_numpy(v).pin_memory() for k, v in cols.items()}
    del cols
    ranged("q1_fission_sf10", lambda: R.q1_fission_run(hw, 1 << 22, st), 38 * N)
    enc, s = R.q1_encode({k: v.cuda() for k, v in hw.items()})
    assert int(s.item()) == 0
    del hw
    hn = {k: v.cpu().pin_memory() for k, v in enc.items()}
    del enc
    ranged("q1n_fission_sf10", lambda: R.q1_narrow_fission_run(hn, 1 << 23, st), 11 * N)


if __name__ == "__main__":
    main()
