"""f2 M=2 timing over predicate pairs with the same output sizes (dev tool):
identical, complementary, overlapping; and the output arrays' relative placement."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda")
ragen.int32_column_dev(2, x)
big = torch.empty(2 * n + (1 << 22), dtype=torch.int32, device="cuda")


def t(chains, outs):
    for _ in range(3):
        R.select_multi(x, chains, outs=outs)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        R.select_multi(x, chains, outs=outs)
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / 20


pairs = {
    "identical x<0, x<0": [[("lt", 0)], [("lt", 0)]],
    "complementary x<0, x>=0": [[("lt", 0)], [("ge", 0)]],
    "bench x<0, |x|<2^30": [[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)]],
    "shifted x<0, x<2^31-2^31": [[("lt", 0)], [("ge", -(2**30)), ("lt", 2**30)]],
    "disjoint halves x<-2^30|.., x>=2^30": [[("lt", -(2**30))], [("ge", 2**30)]],
}
for off_b in [int(a) for a in sys.argv[1:]] or [0, 4096, 1052672]:
    o0 = big[:n]
    o1 = big[n + off_b // 4: 2 * n + off_b // 4]
    for name, ch in pairs.items():
        print(f"out1 offset +{off_b} B  {name:40s} {t(ch, [o0, o1]):.4f} ms", flush=True)
