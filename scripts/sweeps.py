"""SURVEY §8(d) sweeps on one B200 (results go to profiles/r<NN>_*.txt).

  d2: fused vs unfused SELECT chain on 2^28 device-resident int32 rows,
      s in {.01,.05,.10,.25,.50,.75,.90} per stage, k in {1,2,3};
      GB/s against the algorithmic bytes (fused 4+4s^k, unfused
      sum_j 4(s^j+s^(j+1)) B/row) and the fused/unfused time ratio next to
      the bytes ratio the paper's argument predicts (DERIVED A.1).
  d4: host-resident chain (2^28 rows pinned, k=2, s=.5) through
      ra_fission_run: chunk_rows 2^20..2^27 x streams 1..4, fused, plus the
      Fig 16 modes.

usage: python scripts/sweeps.py {d2|d4} [out.txt]
Timing: CUDA events on the current stream, warm-up first, median of reps.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
import ragen  # noqa: E402


def ev_ms(fn, reps=10, warm=3):
    """Mean ms per call over `reps` calls enqueued back to back (the GPU
    never idles between calls, so host launch overhead is not timed)."""
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    b.synchronize()
    return a.elapsed_time(b) / reps


def d2(out):
    n = 1 << 28
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(2, x)
    o = torch.empty(n, dtype=torch.int32, device="cuda")
    out.write("# d2: fused vs unfused SELECT chain, 2^28 int32 rows device-resident, 1x B200\n")
    out.write("# GB/s = algorithmic bytes / kernel time (fused 4+4s^k, unfused sum_j 4(s^j+s^(j+1)) B/row)\n")
    out.write(f"{'s':>5} {'k':>2} {'kept':>10} {'fused_ms':>9} {'fused_GB/s':>10} {'unfused_ms':>10} "
              f"{'unf_GB/s':>9} {'speedup':>8} {'bytes_ratio':>11}\n")
    for s in (0.01, 0.05, 0.10, 0.25, 0.50, 0.75, 0.90):
        for k in (1, 2, 3):
            preds = [("lt", t) for t in ragen.nested_thresholds(s, k)]
            cnt = [None]

            def f():
                cnt[0] = R.select_chain(x, preds, fused=True, out=o)[1]

            def u():
                R.select_chain(x, preds, fused=False, out=o)

            fm = ev_ms(f)
            kept = int(cnt[0].item())
            um = ev_ms(u) if k > 1 else fm
            fb = 4 + 4 * s ** k
            ub = sum(4 * (s ** j + s ** (j + 1)) for j in range(k))
            out.write(f"{s:5.2f} {k:2d} {kept:10d} {fm:9.4f} {fb * n / fm / 1e6:10.0f} {um:10.4f} "
                      f"{ub * n / um / 1e6:9.0f} {um / fm:8.2f} {ub / fb:11.2f}\n")
            out.flush()


def d4(out):
    n = 1 << 28
    preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(4, x)
    h_in = torch.empty(n, dtype=torch.int32, pin_memory=True)
    h_in.copy_(x.cpu())
    del x
    h_out = torch.empty(n, dtype=torch.int32, pin_memory=True)
    h_cnt = torch.zeros(1 << 8, dtype=torch.int64, pin_memory=True)
    streams = [torch.cuda.Stream() for _ in range(4)]
    # pinned copy peak (the paper's Fig 4(b) method)
    d = torch.empty(n, dtype=torch.int32, device="cuda")
    h2d = ev_ms(lambda: d.copy_(h_in, non_blocking=True), 5, 2)
    d2h = ev_ms(lambda: h_out.copy_(d, non_blocking=True), 5, 2)
    del d
    out.write("# d4: host-resident chain (2^28 int32 pinned, k=2, s=.5/stage) through ra_fission_run, 1x B200\n")
    out.write(f"# pinned cudaMemcpy: H2D {4 * n / h2d / 1e6:.1f} GB/s, D2H {4 * n / d2h / 1e6:.1f} GB/s "
              f"(1 GiB each)\n")
    out.write(f"{'mode':>14} {'chunk':>6} {'S':>2} {'ms':>8} {'Grows/s':>8} {'H2D GB/s':>9} {'%H2D_peak':>9}\n")

    def run(chunk, S, fused):
        return ev_ms(lambda: R.fission_run(h_in, preds, chunk, streams[:S], fused=fused, h_out=h_out,
                                           h_chunk_counts=h_cnt), 3, 1)

    def line(mode, chunk, S, fused):
        ms = run(chunk, S, fused)
        lg = chunk.bit_length() - 1
        out.write(f"{mode:>14} {'2^%d' % lg:>6} {S:2d} {ms:8.2f} {n / ms / 1e6:8.2f} {4 * n / ms / 1e6:9.1f} "
                  f"{100 * h2d / ms:9.1f}\n")
        out.flush()

    for mode, chunk, S, fused in (("serial", n, 1, False), ("fusion_only", n, 1, True),
                                  ("fission_only", 1 << 24, 3, False), ("fusion_fission", 1 << 24, 3, True)):
        line(mode, chunk, S, fused)
    for lg in range(20, 28):
        for S in (1, 2, 3, 4):
            line("fused", 1 << lg, S, True)


if __name__ == "__main__":
    what = sys.argv[1]
    f = open(sys.argv[2], "w") if len(sys.argv) > 2 else sys.stdout
    {"d2": d2, "d4": d4}[what](f)
