"""f2 sweep: ra_select_multi (one read, two outputs) vs two single-output
select kernels, 2^28 int32 rows on one GPU, per selectivity pair (dev tool)."""
import sys
import torch
sys.path.insert(0, ".")
import ragen, paper_conf_ipps_wudwcyc12_b200 as R

n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda")
ragen.int32_column_dev(2, x)


def t(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    b.synchronize()
    return a.elapsed_time(b) / reps


outs = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(2)]
print("s0    s1    fused_ms  separate_ms  separate/fused")
for s0, s1 in [(0.01, 0.01), (0.1, 0.1), (0.25, 0.25), (0.1, 0.5), (0.5, 0.5), (0.25, 0.75), (0.9, 0.9)]:
    ch = [[("lt", ragen.nested_thresholds(s0, 1)[0])], [("gt", -ragen.nested_thresholds(s1, 1)[0])]]
    f = t(lambda: R.select_multi(x, ch, outs=outs))
    sp = t(lambda: (R.select_chain(x, ch[0], out=outs[0]), R.select_chain(x, ch[1], out=outs[1])))
    print(f"{s0:<5} {s1:<5} {f:9.4f} {sp:12.4f} {sp / f:10.3f}", flush=True)
