"""ncu driver: select_multi M=2 on 2^28 rows, predicate pair by name (identical | complementary)."""
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
outs = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(2)]
ch = {"identical": [[("lt", 0)], [("lt", 0)]], "complementary": [[("lt", 0)], [("ge", 0)]]}[sys.argv[1]]
for _ in range(4):
    R.select_multi(x, ch, outs=outs)
torch.cuda.synchronize()
