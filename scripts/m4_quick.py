"""f2 M=3/4 quick timing on the bench chains and a few shapes (dev tool; RA_LIB_PATH picks a variant)."""
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
B = [[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)], [("ge", 2**30)], [("lt", -(2**30))]]
cases = {"m4bench": B, "m3bench": B[:3], "m2bench": B[:2], "m4 .01": [[("lt", ragen.nested_thresholds(0.01, 1)[0])]] * 4,
         "m4 .9": [[("lt", ragen.nested_thresholds(0.9, 1)[0])]] * 4, "m1 .25": [[("lt", ragen.nested_thresholds(0.25, 1)[0])]],
         "m1 .01": [[("lt", ragen.nested_thresholds(0.01, 1)[0])]], "m1 .9": [[("lt", ragen.nested_thresholds(0.9, 1)[0])]]}
res = []
for name, ch in cases.items():
    M = len(ch)
    for _ in range(3):
        R.select_multi(x, ch, outs=outs[:M])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        R.select_multi(x, ch, outs=outs[:M])
    e1.record()
    e1.synchronize()
    res.append(f"{name}:{e0.elapsed_time(e1) / 10:.4f}")
print(os.path.basename(os.environ.get("RA_LIB_PATH", "libra.so")), " ".join(res), flush=True)
