"""M=1 select_multi at 2^28 rows over selectivities: output checked against
torch.masked_select on the device, then timed (dev tool; RA_LIB_PATH picks a variant)."""
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
out = torch.empty(n, dtype=torch.int32, device="cuda")
res = []
for s in (0.01, 0.1, 0.25, 0.5, 0.75, 0.9):
    T = ragen.nested_thresholds(s, 1)[0]
    ch = [[("lt", T)]]
    _, cnt = R.select_multi(x, ch, outs=[out])
    exp = torch.masked_select(x, x < T)
    c = int(cnt[0])
    ok = c == exp.numel() and bool(torch.equal(out[:c], exp))
    for _ in range(3):
        R.select_multi(x, ch, outs=[out])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        R.select_multi(x, ch, outs=[out])
    e1.record()
    e1.synchronize()
    res.append(f"s{s}:{e0.elapsed_time(e1) / 20:.4f}{'' if ok else '(WRONG)'}")
    print(os.path.basename(os.environ.get("RA_LIB_PATH", "libra.so")), res[-1], flush=True)
print(os.path.basename(os.environ.get("RA_LIB_PATH", "libra.so")), " ".join(res), flush=True)
