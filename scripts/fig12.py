"""The paper's Fig 12 experiment (§IV-A) on B200 (dev tool).

  old      one SELECT (50% kept) over N rows with the full grid
  new      the same with half the CTAs (RA_SEL_MAX_CTAS)
  stream   two independent SELECTs over N/2 rows each, each with half the CTAs,
           concurrently on two streams (N = total rows of both)
  serial   the two N/2 SELECTs with the full grid, one after the other
  fused    both SELECTs on ONE N/2-row input through ra_select_multi (one read):
           what Fig 2(c)'s pattern buys when the two SELECTs share their input
Each variant is captured once in a CUDA graph (50 repetitions) and replayed, so
host launch overhead does not enter; rows/s = N / time.  Run twice by the GPU
script: full grid and half grid (RA_SEL_MAX_CTAS, read once per process).
"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

mode = sys.argv[1]  # "full" or "half"
REPS = 50


def graph_ms(body):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        body()  # warm-up (workspaces, attributes) outside the capture
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):  # same stream as the warm-up: the cached workspaces are reused
        for _ in range(REPS):
            body()
    g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    g.replay()
    b.record()
    b.synchronize()
    return a.elapsed_time(b) / REPS


for lg in range(20, 29):
    N = 1 << lg
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(1, x)
    a, b = x[:N // 2], x[N // 2:]
    o = [torch.empty(N, dtype=torch.int32, device="cuda") for _ in range(2)]
    s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
    p = [("lt", 0)]

    def one():
        R.select_chain(x, p, out=o[0])

    def two_streams():
        cur = torch.cuda.current_stream()
        s0.wait_stream(cur)
        s1.wait_stream(cur)
        R.select_chain(a, p, out=o[0], stream=s0)
        R.select_chain(b, p, out=o[1], stream=s1)
        cur.wait_stream(s0)
        cur.wait_stream(s1)

    old = graph_ms(one)
    st = graph_ms(two_streams)
    if mode == "full":
        ser = graph_ms(lambda: (R.select_chain(a, p, out=o[0]), R.select_chain(b, p, out=o[1])))
        fu = graph_ms(lambda: R.select_multi(a, [p, [("ge", 0)]], outs=o))
        print(f"full 2^{lg} old_ms {old:.4f} stream_fullgrid_ms {st:.4f} serial_ms {ser:.4f} "
              f"fused_same_input_ms {fu:.4f}", flush=True)
    else:
        print(f"half 2^{lg} new_ms {old:.4f} stream_ms {st:.4f}", flush=True)
