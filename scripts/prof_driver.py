"""Small driver for ncu: runs the hot-path kernels a few times at bench sizes.

usage: python scripts/prof_driver.py {select|unfused|rows|sparse|multi|q1|q1sf100|q1n|q1nsf100|q1time|select1m}
       [reps] [log2n] [k] [sel]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
import ragen  # noqa: E402


def main():
    what = sys.argv[1]
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    log2n = int(sys.argv[3]) if len(sys.argv) > 3 else 28
    k = int(sys.argv[4]) if len(sys.argv) > 4 else 2
    sel = float(sys.argv[5]) if len(sys.argv) > 5 else 0.5
    torch.cuda.set_device(0)
    if what in ("select", "unfused", "select1m"):
        n = 1 << (20 if what == "select1m" else log2n)
        x = torch.empty(n, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(2, x)
        preds = [("lt", t) for t in ragen.nested_thresholds(sel, k)] if what != "select1m" else [("lt", 0)]
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        for _ in range(reps):
            R.select_chain(x, preds, fused=(what != "unfused"), out=out)
    elif what == "q1time":  # CUDA-event timing of the fused Q1 at SF10 and SF100
        for sf in (10, 100):
            n = ragen.rows_for_sf(sf)
            cols = {name: torch.empty(n, dtype=getattr(torch, np.dtype(dt).name), device="cuda")
                    for name, dt in ragen.LINEITEM_COLUMNS}
            ragen.lineitem_dev(5, ragen.parts_for_sf(sf), cols)
            for _ in range(3):
                R.q1(cols)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(reps):
                R.q1(cols)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / reps
            print(f"q1 SF{sf}: {ms:.4f} ms  {38 * n / ms / 1e6:.1f} GB/s  {n / ms * 1e3:.3e} rows/s")
            enc, _ = R.q1_encode(cols)
            del cols
            torch.cuda.empty_cache()
            for _ in range(3):
                R.q1_narrow(enc)
            e0.record()
            for _ in range(reps):
                R.q1_narrow(enc)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / reps
            print(f"q1 narrow SF{sf}: {ms:.4f} ms  {11 * n / ms / 1e6:.1f} GB/s  {n / ms * 1e3:.3e} rows/s")
            cols = enc
            torch.cuda.empty_cache()
    elif what == "rows":  # tuple SELECT (f3): key + two int32 fields, chain k at sel
        n = 1 << log2n
        x = torch.empty(n, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(2, x)
        f1 = torch.empty(n, dtype=torch.int32, device="cuda")
        f2 = torch.empty(n, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(102, f1)
        ragen.int32_column_dev(103, f2)
        preds = [("lt", t) for t in ragen.nested_thresholds(sel, k)]
        for _ in range(reps):
            R.select_rows(x, preds, [x, f1, f2], rowids=False)
    elif what == "q1n":  # narrow Q1 at SF10 (for ncu)
        n = ragen.rows_for_sf(10)
        cols = {name: torch.empty(n, dtype=getattr(torch, np.dtype(dt).name), device="cuda")
                for name, dt in ragen.LINEITEM_COLUMNS}
        ragen.lineitem_dev(5, ragen.parts_for_sf(10), cols)
        enc, _ = R.q1_encode(cols)
        for _ in range(reps):
            R.q1_narrow(enc)
    elif what in ("q1", "q1sf100", "q1nsf100"):
        sf = 10 if what == "q1" else 100
        n = ragen.rows_for_sf(sf)
        cols = {name: torch.empty(n, dtype=getattr(torch, np.dtype(dt).name), device="cuda")
                for name, dt in ragen.LINEITEM_COLUMNS}
        ragen.lineitem_dev(5, ragen.parts_for_sf(sf), cols)
        if what == "q1nsf100":
            cols, _ = R.q1_encode(cols)
            torch.cuda.empty_cache()
        for _ in range(reps):
            (R.q1_narrow if what == "q1nsf100" else R.q1)(cols)
    elif what == "multi1":  # the multi kernel with one output (M = 1) at selectivity sel
        n = 1 << log2n
        x = torch.empty(n, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(2, x)
        ch = [[("lt", ragen.nested_thresholds(sel, 1)[0])]]
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        for _ in range(reps):
            R.select_multi(x, ch, outs=[out])
    elif what == "multi":  # f2: M outputs on one 2^log2n column, the bench's chains (M = k arg)
        n = 1 << log2n
        x = torch.empty(n, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(2, x)
        chains = [[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)], [("ge", 2**30)], [("lt", -(2**30))]][:k]
        if sel > 0.5:  # dense pair: both outputs keep ~sel
            t = int(-(2**31) + sel * 2**32)
            chains = [[("lt", t)], [("gt", -t)]][:k]
        outs = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in chains]
        for _ in range(reps):
            R.select_multi(x, chains, outs=outs)
    elif what == "sparse":  # f3 sparse path: 3 int32 fields, no caller ids (key pass + ids_kernel + gather_kernel)
        n = 1 << log2n
        x = torch.empty(n, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(2, x)
        f1 = torch.empty(n, dtype=torch.int32, device="cuda")
        f2 = torch.empty(n, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(102, f1)
        ragen.int32_column_dev(103, f2)
        preds = [("lt", t) for t in ragen.nested_thresholds(sel, k)]
        for _ in range(reps):
            R.select_rows(x, preds, [x, f1, f2], rowids=False)
    torch.cuda.synchronize()
    print("done", what)


if __name__ == "__main__":
    main()
