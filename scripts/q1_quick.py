"""Quick Q1 timing, wide and narrow, SF10 and SF100 on one GPU, back-to-back
launches (dev tool; RA_LIB_PATH picks a variant build).  Prints ms per launch
and a hash of the finalized rows (equal across variants = same result)."""
import hashlib
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

out = []
for sf in (10, 100):
    N = ragen.rows_for_sf(sf)
    cols = {name: torch.empty(N, dtype=getattr(torch, np.dtype(dt).name), device="cuda")
            for name, dt in ragen.LINEITEM_COLUMNS}
    ragen.lineitem_dev(7, ragen.parts_for_sf(sf), cols)
    part = torch.zeros(400, dtype=torch.uint8, device="cuda")
    enc, _ = R.q1_encode(cols)
    for name, fn in (("wide", lambda: R.q1(cols, partial=part)), ("narrow", lambda: R.q1_narrow(enc, partial=part))):
        for _ in range(5):
            fn()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(30):
            fn()
        e1.record()
        e1.synchronize()
        rows, rc = R.q1_finalize(bytes(part.cpu().numpy().tobytes()))
        h = hashlib.sha1(repr(rows).encode()).hexdigest()[:8]
        out.append(f"SF{sf}/{name}:{e0.elapsed_time(e1) / 30:.4f}({h},rc{rc})")
    del cols, enc
    torch.cuda.empty_cache()
print(os.path.basename(os.environ.get("RA_LIB_PATH", "libra.so")), " ".join(out), flush=True)
