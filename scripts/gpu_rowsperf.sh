mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout 900 python -m pytest tests/test_select_rows_gpu.py -x -q > gpurun_out/pytest_rows.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_rows.log
python - <<'PY'
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_wudwcyc12_b200 as R, ragen
n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(2, x)
f1 = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(102, f1)
f2 = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(103, f2)
for s, k in ((0.5, 2), (0.5, 1), (0.01, 1), (0.9, 1)):
    p = [("lt", t) for t in ragen.nested_thresholds(s, k)]
    for fields in ([x], [x, f1, f2]):
        for _ in range(3): R.select_rows(x, p, fields, rowids=False)
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True); e0.record()
        for _ in range(10): _, _, c = R.select_rows(x, p, fields, rowids=False)
        e1.record(); e1.synchronize(); ms = e0.elapsed_time(e1) / 10
        kk = int(c.item())
        print(f"s={s} k={k} fields={len(fields)} ms={ms:.4f} alg GB/s={(4*n + 8*kk*len(fields))/ms/1e6:.0f}")
PY
