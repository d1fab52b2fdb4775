"""Dev tool: locate SELECT mismatches vs the oracle at several sizes."""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ipps_wudwcyc12_b200 as R, ragen, oracle
for lg, s, k in ((22, .5, 2), (24, .5, 2), (24, .1, 1), (24, .9, 1), (26, .5, 2)):
    n = 1 << lg
    x = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(2, x)
    preds = [("lt", t) for t in ragen.nested_thresholds(s, k)]
    out, c = R.select_chain(x, preds); torch.cuda.synchronize(); c = int(c.item())
    exp = oracle.select(x.cpu().numpy(), preds)
    got = out[:c].cpu().numpy()
    bad = np.nonzero(got[:min(c, exp.size)] != exp[:min(c, exp.size)])[0]
    msg = f"n=2^{lg} s={s} k={k}: count {c} vs {exp.size}, mismatches {bad.size}"
    if bad.size:
        # map first bad output position to the source tile via the oracle's selected index
        m = np.nonzero(np.all([x.cpu().numpy() < t for t in ragen.nested_thresholds(s, k)], axis=0))[0]
        tiles = np.unique(m[bad] // 8192)
        msg += f", tiles {tiles[:10]} ... ({tiles.size} tiles), cta {np.unique(tiles % 296)[:10]}, round {np.unique(tiles // 296)[:10]}"
    print(msg, flush=True)
