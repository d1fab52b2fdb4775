"""Per-CTA %globaltimer stamps of q1n_kernel (needs the RA_Q1N_TIMES build:
make variant NAME=qnt FLAGS=-DRA_Q1N_TIMES; RA_LIB_PATH=build/libra_qnt.so).
Stamps: 0 entry, 1 after griddepcontrol.wait, 2 after init, 3 compute loop
done (warp 0), 4 final flush done, 5 CTA partial written, 6 after the grid fold."""
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

N = ragen.rows_for_sf(10)
cols = {name: torch.empty(N, dtype=getattr(torch, np.dtype(dt).name), device="cuda") for name, dt in ragen.LINEITEM_COLUMNS}
ragen.lineitem_dev(7, ragen.parts_for_sf(10), cols)
enc, _ = R.q1_encode(cols)
del cols
part = torch.zeros(400, dtype=torch.uint8, device="cuda")
buf = (ctypes.c_ulonglong * (1184 * 16))()
for m in (1 << 20, N):
    nc = {k: v[:m] for k, v in enc.items()}
    for mode in ("single", "b2b"):
        for _ in range(3):
            R.q1_narrow(nc, partial=part)
        torch.cuda.synchronize()
        if mode == "b2b":
            for _ in range(5):
                R.q1_narrow(nc, partial=part)
        else:
            R.q1_narrow(nc, partial=part)
        torch.cuda.synchronize()
        _ra._lib.raqn_times(buf)
        t = np.frombuffer(buf, dtype=np.uint64).reshape(1184, 16)[:148].astype(np.int64)
        t0 = t[:, 0].min()
        rel = (t[:, :7] - t0) / 1000.0
        print(f"rows {m} ({mode}, last launch): us since the first CTA entered; min / median / max over CTAs")
        for k, name in enumerate(["entry", "dep_wait", "init", "loop_done", "flush_done", "partial", "fold_done"]):
            print(f"   {name:10s} {rel[:, k].min():8.2f} {np.median(rel[:, k]):8.2f} {rel[:, k].max():8.2f}")
        last = int(np.argmax(rel[:, 6]))
        print(f"   last CTA {last} on SM {t[last, 7]}: {rel[last, :7].round(2).tolist()}")
        slow = int(np.argmax(rel[:, 3]))
        print(f"   slowest loop CTA {slow} on SM {t[slow, 7]}: {rel[slow, :7].round(2).tolist()}", flush=True)
