"""Per-CTA %globaltimer stamps of select_multi_kernel (needs the RA_MO_TIMES
build: make variant NAME=mot FLAGS=-DRA_MO_TIMES; RA_LIB_PATH=build/libra_mot.so).
Stamps: 0 entry, 1 after griddepcontrol.wait, 2 after init, 3 producer drew
past the last tile, 4 first tile in smem (group 0), 5 compute saw the end,
6 look-back warps done, 7 writers done."""
import ctypes
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
from paper_conf_ipps_wudwcyc12_b200 import _ra  # noqa: E402

n = 1 << 28
x = torch.empty(n, dtype=torch.int32, device="cuda")
ragen.int32_column_dev(2, x)
out = torch.empty(n, dtype=torch.int32, device="cuda")
buf = (ctypes.c_ulonglong * (2048 * 16))()
NAMES = ["entry", "dep_wait", "init", "last_ticket", "first_tile", "compute_end", "lookback_end", "writers_end"]
for label, preds in (("k2 s.5 (headline)", [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]),
                     ("k1 s.01", [("lt", ragen.nested_thresholds(0.01, 1)[0])])):
    for mode in ("single", "b2b"):
        for _ in range(3):
            R.select_chain(x, preds, out=out)
        torch.cuda.synchronize()
        for _ in range(5 if mode == "b2b" else 1):
            R.select_chain(x, preds, out=out)
        torch.cuda.synchronize()
        _ra._lib.ramo_times(buf)
        t = np.frombuffer(buf, dtype=np.uint64).reshape(2048, 16)[:148].astype(np.int64)
        t0 = t[:, 0].min()
        rel = (t[:, :8] - t0) / 1000.0
        print(f"{label} ({mode}, last launch): us since the first CTA entered; min / median / max over CTAs")
        for k, name in enumerate(NAMES):
            print(f"   {name:13s} {rel[:, k].min():8.2f} {np.median(rel[:, k]):8.2f} {rel[:, k].max():8.2f}")
        last = int(np.argmax(rel[:, 7]))
        print(f"   last CTA {last} (SM {t[last, 8]}): {rel[last].round(2).tolist()}", flush=True)
