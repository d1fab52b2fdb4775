# tuple SELECT: payload compaction (default) vs the id gather (RA_TUPLE_GATHER=1), 2^28 rows, 3 int32 fields
mkdir -p gpurun_out
make -s all 2>&1 | grep -iE "error" ; true
timeout 600 python -m pytest tests/test_select_rows_gpu.py -x -q 2>&1 | tail -3
cat > /tmp/rows_ab.py <<'PY'
import sys, torch, numpy as np
sys.path.insert(0, ".")
import ragen, paper_conf_ipps_wudwcyc12_b200 as R
n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(2, x)
f = [x] + [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(2)]
ragen.int32_column_dev(102, f[1]); ragen.int32_column_dev(103, f[2])
f8 = torch.empty(n, dtype=torch.int64, device="cuda"); f8.copy_(f[1])
for _ in range(5): R.select_rows(x, [("lt", 0)], f, rowids=True); R.select_rows(x, [("lt", 0)], [f8], rowids=False)
torch.cuda.synchronize()
for name, preds in [("s=.01", [("lt", -2104533975)]), ("s=.03", [("lt", -2018634629)]), ("s=.05", [("lt", -1932735283)]), ("s=.1", [("lt", -1717986918)]), ("s=.25", [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]),
                    ("s=.5", [("lt", 0)]), ("s=.9", [("lt", 1717986918)])]:
    for label, pays in [("3xi32", f), ("1xi64", [f8])]:
        for rid in (False, True):
            for _ in range(3): R.select_rows(x, preds, pays, rowids=rid)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(10): ids, outs, cnt = R.select_rows(x, preds, pays, rowids=rid)
            e1.record(); e1.synchronize()
            print(f"{name} {label} rowids={int(rid)}  ms {e0.elapsed_time(e1)/10:.4f}  count {int(cnt.item())}", flush=True)
PY
( echo "== device choice (gather below 1/32 [4-B fields] or 1/8 [8-B] selected, else streaming compaction)"
  timeout 300 python /tmp/rows_ab.py
  echo "== RA_TUPLE_GATHER=1 (id gather always)"
  RA_TUPLE_GATHER=1 timeout 300 python /tmp/rows_ab.py ) 2>&1 | tee gpurun_out/rows_ab.txt
