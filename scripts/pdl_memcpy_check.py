"""Does a kernel launched with programmatic stream serialization wait for an
H2D copy that precedes it on the stream?  (dev check; measured on B200: yes,
0 stale reads in 20 tries, profiles/r01_soak.txt)  The device column is
zeroed, a 1 GiB pinned H2D copy refills it asynchronously, and the select
kernel follows at once: a stale read shows up as a wrong count."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
import ragen  # noqa: E402

n = 1 << 28
h = torch.empty(n, dtype=torch.int32, pin_memory=True)
ragen.int32_column(3, n, out=h.numpy())
exp = int((h.numpy() < 0).sum())
x = torch.empty(n, dtype=torch.int32, device="cuda")
bad = 0
for it in range(20):
    x.fill_(5)  # every row fails "x < 0" until the copy lands
    torch.cuda.synchronize()
    x.copy_(h, non_blocking=True)
    out, c = R.select_chain(x, [("lt", 0)])
    torch.cuda.synchronize()
    if int(c.item()) != exp:
        bad += 1
        print("iter", it, "count", int(c.item()), "expected", exp, flush=True)
print("stale reads:", bad, "of 20")
