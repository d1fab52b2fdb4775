"""tuple SELECT (ra_select_rows), 2^28 rows: device choice vs the id gather
(RA_TUPLE_GATHER=1), outputs and workspace preallocated, each configuration
warmed up before it is timed (dev tool; scripts/gpu_rows_ab.sh)."""
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
f = [x] + [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(2)]
ragen.int32_column_dev(102, f[1])
ragen.int32_column_dev(103, f[2])
f8 = torch.empty(n, dtype=torch.int64, device="cuda")
f8.copy_(f[1])
ids = torch.empty(n, dtype=torch.uint32, device="cuda")
outs4 = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(3)]
out8 = torch.empty(n, dtype=torch.int64, device="cuda")
cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
wsb = R.ra_select_rows_workspace_bytes(n, 2)
ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
sh = int(torch.cuda.current_stream().cuda_stream)
for name, preds in [("s=.01", [("lt", -2104533975)]), ("s=.03", [("lt", -2018634629)]),
                    ("s=.05", [("lt", -1932735283)]), ("s=.1", [("lt", -1717986918)]),
                    ("s=.25", [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]), ("s=.5", [("lt", 0)]),
                    ("s=.9", [("lt", 1717986918)])]:
    P = R.make_preds(preds)
    for label, cols, outs in [("3xi32", f, outs4), ("1xi64", [f8], [out8])]:
        pl = (R.ra_payload * len(cols))()
        for j, (c, o) in enumerate(zip(cols, outs)):
            pl[j].col, pl[j].out, pl[j].elem_bytes = c.data_ptr(), o.data_ptr(), c.element_size()
        for rid in (False, True):
            args = (x.data_ptr(), n, P, len(preds), ids.data_ptr() if rid else 0, pl, len(cols), n, cnt.data_ptr(),
                    ws.data_ptr(), wsb, sh)
            for _ in range(3):
                R.ra_select_rows(*args)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(10):
                R.ra_select_rows(*args)
            e1.record()
            e1.synchronize()
            print(f"{name} {label} rowids={int(rid)}  ms {e0.elapsed_time(e1) / 10:.4f}  count {int(cnt.item())}",
                  flush=True)
