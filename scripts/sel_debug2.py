"""Dev tool: inspect one corrupted tile's output run."""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ipps_wudwcyc12_b200 as R, ragen, oracle
n = 1 << 24; s, k = .5, 2
x = torch.empty(n, dtype=torch.int32, device="cuda"); ragen.int32_column_dev(2, x)
preds = [("lt", t) for t in ragen.nested_thresholds(s, k)]
xh = x.cpu().numpy()
for rep in range(3):
    out, c = R.select_chain(x, preds); torch.cuda.synchronize(); c = int(c.item())
    exp = oracle.select(xh, preds); got = out[:c].cpu().numpy()
    sel = np.nonzero(np.all([xh < t for t in ragen.nested_thresholds(s, k)], axis=0))[0]
    tile_of = sel // 8192
    bad = np.nonzero(got != exp)[0]
    print("rep", rep, "mismatches", bad.size, "tiles", np.unique(tile_of[bad]))
    for t in np.unique(tile_of[bad])[:3]:
        idx = np.nonzero(tile_of == t)[0]; a, b = idx[0], idx[-1] + 1
        g = got[a:b]; e = exp[a:b]
        nb = np.nonzero(g != e)[0]
        print(f"  tile {t}: out[{a}:{b}] ({b-a} rows), bad local {nb[:5]}..{nb[-5:]} ({nb.size})")
        # where do the wrong values come from?
        pos = {v: i for i, v in enumerate(exp)}
        src = [pos.get(v, -1) for v in g[nb[:8]]]
        print("    wrong values found at exp positions", src, "-> tiles", [tile_of[p] if p >= 0 else None for p in src])
