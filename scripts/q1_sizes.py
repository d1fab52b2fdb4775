"""Q1 (wide and narrow) time vs table size, back-to-back launches and single
launches (dev tool): separates a per-launch fixed cost from the per-row rate."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

N = ragen.rows_for_sf(40)
cols = {name: torch.empty(N, dtype=getattr(torch, np.dtype(dt).name), device="cuda") for name, dt in ragen.LINEITEM_COLUMNS}
ragen.lineitem_dev(7, ragen.parts_for_sf(40), cols)
enc, _ = R.q1_encode(cols)
part = torch.zeros(400, dtype=torch.uint8, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
print("rows       wide_b2b  wide_single  narrow_b2b  narrow_single  (ms)")
for m in (1 << 20, 1 << 22, 1 << 24, 15_000_000, 30_000_000, 60_000_000, 120_000_000, 240_000_000):
    wc = {k: v[:m] for k, v in cols.items()}
    nc = {k: v[:m] for k, v in enc.items()}
    res = []
    for fn in (lambda: R.q1(wc, partial=part), lambda: R.q1_narrow(nc, partial=part)):
        for _ in range(3):
            fn()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            fn()
        e1.record()
        e1.synchronize()
        b2b = e0.elapsed_time(e1) / 20
        singles = []
        for _ in range(10):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            b.synchronize()
            singles.append(a.elapsed_time(b))
        res += [b2b, float(np.median(singles))]
    print(f"{m:11d} {res[0]:9.4f} {res[1]:11.4f} {res[2]:11.4f} {res[3]:13.4f}", flush=True)
