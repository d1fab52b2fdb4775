"""f2 sweep (dev tool): ra_select_multi (ONE read of the input, M outputs) vs M
single-output select kernels (M reads), 2^28 int32 rows on one GPU; and M = 1
through the multi kernel vs ra_select_chain (the single-output kernel).
Algorithmic bytes: 4n read + 4 * sum(counts) written (fused); prints GB/s and
the fraction of MEASURED_PEAKS.json hbm_gbs."""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda")
ragen.int32_column_dev(2, x)


def t(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    b.synchronize()
    return a.elapsed_time(b) / reps


def lt(s):
    return [("lt", ragen.nested_thresholds(s, 1)[0])] if s < 1 else [("ge", -(2**31))]


def gt(s):
    return [("gt", -ragen.nested_thresholds(s, 1)[0])] if s < 1 else [("ge", -(2**31))]


outs = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
print(f"# 2^28 int32 rows, one B200; peak = {PEAK} GB/s (MEASURED_PEAKS.json hbm_gbs)")
print("M  sel                      fused_ms  GB/s    frac  | separate_ms  separate/fused")
cases = [(1, (s,)) for s in (0.01, 0.1, 0.25, 0.5, 0.75, 0.9)]
cases += [(2, p) for p in [(0.01, 0.01), (0.1, 0.1), (0.25, 0.25), (0.1, 0.5), (0.5, 0.5), (0.25, 0.75), (0.9, 0.9)]]
cases += [(3, p) for p in [(0.01, 0.01, 0.01), (0.25, 0.25, 0.25), (0.5, 0.5, 0.5), (0.9, 0.9, 0.9)]]
cases += [(4, p) for p in [(0.01,) * 4, (0.25,) * 4, (0.5, 0.5, 0.25, 0.25), (0.5,) * 4, (0.9,) * 4]]
for M, sel in cases:
    ch = [(lt if o % 2 == 0 else gt)(s) for o, s in enumerate(sel)]
    cnt = None

    def fused():
        global cnt
        _, cnt = R.select_multi(x, ch, outs=outs[:M])
    f = t(fused)
    kept = sum(int(c) for c in cnt.cpu().tolist()[:M])
    if os.environ.get("MS_FUSED_ONLY"):
        print(f"{M}  {str(sel):24s} {f:8.4f}", flush=True)
        continue
    sp = t(lambda: [R.select_chain(x, ch[o], out=outs[o]) for o in range(M)])
    gbs = (4 * n + 4 * kept) / (f * 1e-3) / 1e9
    print(f"{M}  {str(sel):24s} {f:8.4f} {gbs:7.0f} {gbs / PEAK:6.3f}  | {sp:10.4f} {sp / f:10.3f}", flush=True)
