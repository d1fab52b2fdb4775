# one tuple-SELECT configuration, for ncu launch lists (dev tool)
import sys
import torch
sys.path.insert(0, ".")
import ragen, paper_conf_ipps_wudwcyc12_b200 as R
n = 1 << 28
thr = int(sys.argv[1]) if len(sys.argv) > 1 else 0
x = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(2, x)
f = [x] + [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(2)]
ragen.int32_column_dev(102, f[1]); ragen.int32_column_dev(103, f[2])
for _ in range(3):
    ids, outs, cnt = R.select_rows(x, [("lt", thr)], f, rowids=False)
torch.cuda.synchronize()
print(int(cnt.item()))
