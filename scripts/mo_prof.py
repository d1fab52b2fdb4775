"""select_multi per-wait cycle profile (needs the RA_MO_PROFILE build:
make variant NAME=prof FLAGS=-DRA_MO_PROFILE; RA_LIB_PATH=build/libra_prof.so)."""
import ctypes
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
from paper_conf_ipps_wudwcyc12_b200 import _ra  # noqa: E402

NAMES = {1: "producer empty wait", 4: "writer placed wait", 5: "writer scattered wait", 6: "compute full wait",
         8: "compute metadata wait", 9: "compute allocd wait", 10: "compute ring wait", 11: "compute iteration",
         12: "compute B1", 13: "compute gtid0 section", 14: "compute B2", 15: "compute scatter",
         16: "writer write", 17: "look-back window sums", 18: "count -> placed", 19: "placed -> written",
         20: "window issue -> resolve", 21: "count -> window issue", 22: "window words (avg)",
         23: "windows read directly (frac)", 24: "re-poll rounds per pass"}
n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda")
ragen.int32_column_dev(2, x)
outs = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
buf = (ctypes.c_ulonglong * 64)()
CASES = {"m1": [(1, 0.01), (1, 0.25)], "dense": [(2, 0.9), (4, 0.9), (4, 0.5)],
         "m2pair": [(2, 0.5), (2, "comp")], "m4bench": [(4, "bench4")]}.get(
    os.environ.get("MO_PROF_CASES", ""), [(1, 0.01), (1, 0.5), (2, 0.5), (2, 0.9), (3, 0.01)])
for M, s in CASES:
    ch = ([[("lt", 0)], [("ge", 0)]] if s == "comp"  # complementary pair
          else [[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)], [("ge", 2**30)], [("lt", -(2**30))]] if s == "bench4"
          else [[("lt", ragen.nested_thresholds(s, 1)[0])]] * M)
    for _ in range(3):
        R.select_multi(x, ch, outs=outs[:M])
    _ra._lib.ramo_prof(buf)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5):
        R.select_multi(x, ch, outs=outs[:M])
    e1.record()
    e1.synchronize()
    _ra._lib.ramo_prof(buf)
    print(f"M={M} s={s}: {e0.elapsed_time(e1) / 5:.4f} ms/launch (profiling build)")
    for c in sorted(NAMES):
        cnt = buf[32 + c]
        if cnt:
            print(f"   {NAMES[c]:26s} {buf[c] / cnt:10.3f} cycles avg  x {cnt / 5:10.0f} per launch (CTA 0)")
