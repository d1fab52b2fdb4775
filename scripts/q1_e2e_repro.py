"""Repeat bench.py's q1_e2e leg (wide + narrow Q1 under fission, SF10) and
compare both with the device-resident result (dev check)."""
import sys
import types

import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
import ragen  # noqa: E402

D = bench.Dist()
args = types.SimpleNamespace()
N = ragen.rows_for_sf(10)
cols = ragen.lineitem(bench.Q1_SEED, N, ragen.parts_for_sf(10))
ref, _ = R.q1_finalize(bytes(R.q1({k: torch.from_numpy(v).cuda() for k, v in cols.items()}).cpu().numpy().tobytes()))
del cols
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 8
fails = 0
for it in range(reps):
    try:
        bench.q1_e2e(args, D, torch, R, 10)
    except AssertionError as e:
        fails += 1
        print("iter", it, "assertion:", e, flush=True)
print("failures", fails, "of", reps)
