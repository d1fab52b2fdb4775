"""Soak test (dev tool): thousands of back-to-back launches of every select
path with random sizes, offsets and selectivities on one stream, each result
checked against numpy (counts + sampled values).  Run under `timeout`."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_wudwcyc12_b200 as R  # noqa: E402
import ragen  # noqa: E402

rng = np.random.default_rng(int(sys.argv[2]) if len(sys.argv) > 2 else 1)
iters = int(sys.argv[1]) if len(sys.argv) > 1 else 2000
base = ragen.int32_column(99, (1 << 22) + 8)
bd = torch.from_numpy(base).cuda()
fstreams = [torch.cuda.Stream() for _ in range(3)]
t0 = time.time()
for it in range(iters):
    n = int(rng.choice([0, 1, 7, 4096, 8192, 8193, 100_003, 1 << 20, (1 << 21) + 3, (1 << 22) - 5]))
    off = int(rng.integers(0, 4))
    x, xd = base[off:off + n], bd[off:off + n]
    t = int(rng.integers(-2**31, 2**31 - 1))
    kind = it % 4
    if kind == 0:
        out, c = R.select_chain(xd, [("lt", t), ("ne", 5)], fused=bool(rng.integers(0, 2)))
        e = x[(x < t) & (x != 5)]
        c = int(c.item())
        assert c == e.size and np.array_equal(out[:c].cpu().numpy(), e), ("chain", it, n, off, t)
    elif kind == 1:  # 1..4 SELECTs on one input, alternating < and > thresholds
        M = int(rng.integers(1, 5))
        ts = [int(rng.integers(-2**31, 2**31 - 1)) for _ in range(M)]
        chains = [[("lt", ts[o])] if o % 2 == 0 else [("gt", ts[o])] for o in range(M)]
        outs, cnt = R.select_multi(xd, chains)
        cs = [int(v) for v in cnt.cpu().tolist()][:M]
        for o in range(M):
            e = x[x < ts[o]] if o % 2 == 0 else x[x > ts[o]]
            assert cs[o] == e.size and np.array_equal(outs[o][:cs[o]].cpu().numpy(), e), ("multi", it, n, off, M, o)
    elif kind == 2:
        ids, outs, c = R.select_rows(xd, [("lt", t)], [xd], rowids=bool(rng.integers(0, 2)))
        e = x[x < t]
        c = int(c.item())
        assert c == e.size and np.array_equal(outs[0][:c].cpu().numpy(), e), ("rows", it, n, off, t)
    else:
        m = max(1, n)
        cols = ragen.lineitem(it, m, 2000)
        dc = {k: torch.from_numpy(v).cuda() for k, v in cols.items()}
        part = R.q1(dc)
        rows, rc = R.q1_finalize(bytes(part.cpu().numpy().tobytes()))
        sel = cols["shipdate"] <= R.Q1_CUTOFF_DELTA90
        assert rc == R.RA_OK and sum(r["count_order"] for r in rows) == int(sel.sum()), ("q1", it, m)
        enc, st = R.q1_encode(dc)  # narrow (f4) must equal wide
        nrows, nrc = R.q1_finalize(bytes(R.q1_narrow(enc).cpu().numpy().tobytes()))
        assert nrc == R.RA_OK and nrows == rows, ("q1 narrow", it, m)
        if it % 16 == 3:  # host-resident under fission (f1), random chunking
            h = {k: torch.from_numpy(v).pin_memory() for k, v in cols.items()}
            S = int(rng.integers(1, 4))
            fr, _ = R.q1_finalize(bytes(R.q1_fission_run(h, int(rng.integers(1, m + 1)), fstreams[:S])))
            assert fr == rows, ("q1 fission", it, m, S)
    if it % 500 == 0:
        print(f"iter {it} ok ({time.time() - t0:.1f} s)", flush=True)
torch.cuda.synchronize()
print(f"soak: {iters} iterations ok in {time.time() - t0:.1f} s")
