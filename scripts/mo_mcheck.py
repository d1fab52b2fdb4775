"""select_multi M = 1..4 on a few sizes, outputs checked against torch.masked_select
(dev tool for variant builds; RA_LIB_PATH picks the build).  Prints one line per case."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ragen  # noqa: E402
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402

B = [[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)], [("ge", 2**30)], [("lt", -(2**30))]]
for n in (3 * 8192 + 5, 1 << 22, 1 << 26):
    x = torch.empty(n, dtype=torch.int32, device="cuda")
    ragen.int32_column_dev(5, x)
    for M in (1, 2, 3, 4):
        ch = B[:M]
        outs, cnt = R.select_multi(x, ch)
        torch.cuda.synchronize()
        ok = True
        for o, c, chain in zip(outs, cnt.cpu().tolist(), ch):
            m = torch.ones(n, dtype=torch.bool, device="cuda")
            for op, t in chain:
                m &= {"lt": x < t, "gt": x > t, "ge": x >= t}[op]
            e = torch.masked_select(x, m)
            ok &= int(c) == e.numel() and bool(torch.equal(o[:int(c)], e))
        print(f"n={n} M={M} {'ok' if ok else 'WRONG'}", flush=True)
