"""Quick select_multi timing at a few shapes (dev tool; RA_LIB_PATH picks a variant build)."""
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
outs = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
res = []
for M, s in [(1, 0.01), (1, 0.25), (1, 0.5), (1, 0.9), (2, 0.5), (2, 0.9), (3, 0.01), (3, 0.5), (4, 0.01), (4, 0.5), (4, 0.9)]:
    ch = [[("lt", ragen.nested_thresholds(s, 1)[0])]] * M
    for _ in range(3):
        R.select_multi(x, ch, outs=outs[:M])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        R.select_multi(x, ch, outs=outs[:M])
    e1.record()
    e1.synchronize()
    res.append(f"M{M}/{s}:{e0.elapsed_time(e1) / 10:.4f}")
for s in (0.01, 0.5, 0.9, 0.25):
    p = [("lt", ragen.nested_thresholds(s, 1)[0])] if s != 0.25 else [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
    for _ in range(3):
        R.select_chain(x, p, out=outs[0])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        R.select_chain(x, p, out=outs[0])
    e1.record()
    e1.synchronize()
    res.append(f"chain{'k2' if s == 0.25 else ''}/{s}:{e0.elapsed_time(e1) / 10:.4f}")
print(os.path.basename(os.environ.get("RA_LIB_PATH", "libra.so")), " ".join(res), flush=True)
