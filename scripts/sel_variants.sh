mkdir -p gpurun_out
for d in 0 1 2 3; do
RA_SEL_DEBUG=$d python - <<'PY'
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_wudwcyc12_b200 as R, ragen
n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device='cuda'); ragen.int32_column_dev(2, x)
preds = [('lt', t) for t in ragen.nested_thresholds(0.5, 2)]
out = torch.empty(n, dtype=torch.int32, device='cuda')
for _ in range(3): R.select_chain(x, preds, out=out)
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record()
for _ in range(20): R.select_chain(x, preds, out=out)
e1.record(); e1.synchronize()
print('dbg', os.environ['RA_SEL_DEBUG'], 'ms', e0.elapsed_time(e1) / 20)
PY
done
