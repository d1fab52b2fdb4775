"""ncu driver: wide and narrow Q1 over the first M rows (default 2^20), a few launches each."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

m = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 20
cols = {name: torch.empty(m, dtype=getattr(torch, np.dtype(dt).name), device="cuda") for name, dt in ragen.LINEITEM_COLUMNS}
ragen.lineitem_dev(7, max(1, m // 6_000_000), cols)
enc, _ = R.q1_encode(cols)
part = torch.zeros(400, dtype=torch.uint8, device="cuda")
for _ in range(3):
    R.q1(cols, partial=part)
    R.q1_narrow(enc, partial=part)
torch.cuda.synchronize()
