"""Fused chain at small n: select_fused_kernel vs select_multi_kernel<1> (dev tool).
Run with RA_SEL_SMALL_ROWS=0 (always the multi pass) and =1e12 (always the
single-output kernel); back-to-back launches and CUDA-graph replay."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

tag = os.environ.get("RA_SEL_SMALL_ROWS", "default")
sh = int(torch.cuda.current_stream().cuda_stream)
for lg in range(16, 27):
    n = 1 << lg
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(1, x)
    out = torch.empty(n, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    wsb = R.ra_select_workspace_bytes(n, 1, 1)
    ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
    P = R.make_preds([("lt", 0)])
    a = (x.data_ptr(), n, P, 1, 1, out.data_ptr(), n, cnt.data_ptr(), ws.data_ptr(), wsb)
    for _ in range(20):
        R.ra_select_chain(*a, sh)
    reps = 200
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        R.ra_select_chain(*a, sh)
    e1.record()
    e1.synchronize()
    b2b = e0.elapsed_time(e1) / reps * 1e3
    print(f"{tag} 2^{lg} back_to_back_us {b2b:.2f} count {int(cnt.item())}", flush=True)
