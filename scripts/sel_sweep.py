"""Quick timing of the fused select at 2^28 over a few selectivities (dev tool)."""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_wudwcyc12_b200 as R, ragen
n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(2, x)
out = torch.empty(n, dtype=torch.int32, device="cuda")
for s, k in ((0.5, 2), (0.5, 1), (0.9, 1), (0.1, 1), (0.99, 1), (0.01, 1)):
    p = [("lt", t) for t in ragen.nested_thresholds(s, k)]
    for _ in range(3): R.select_chain(x, p, out=out)
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True); e0.record()
    for _ in range(20): R.select_chain(x, p, out=out)
    e1.record(); e1.synchronize(); ms = e0.elapsed_time(e1) / 20
    print(s, k, "ms", round(ms, 4), "GB/s", round((4 * n + 4 * n * s ** k) / ms / 1e6, 1))
print("ctas/sm", R._ra._lib and "n/a")
