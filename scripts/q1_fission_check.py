import sys, torch
sys.path.insert(0, ".")
import ragen, paper_conf_ipps_wudwcyc12_b200 as R
N = ragen.rows_for_sf(10)
cols = ragen.lineitem(5, N, ragen.parts_for_sf(10))
h = {k: torch.from_numpy(v).pin_memory() for k, v in cols.items()}
d = {k: v.cuda() for k, v in h.items()}
ref, rc = R.q1_finalize(bytes(R.q1(d).cpu().numpy().tobytes()))
enc, st = R.q1_encode(d)
hn = {k: v.cpu().pin_memory() for k, v in enc.items()}
nd, _ = R.q1_finalize(bytes(R.q1_narrow(enc).cpu().numpy().tobytes()))
print("device wide == device narrow:", nd == ref)
streams = [torch.cuda.Stream() for _ in range(3)]
bad = 0
for it in range(int(sys.argv[1]) if len(sys.argv) > 1 else 30):
    w, _ = R.q1_finalize(bytes(R.q1_fission_run(h, 1 << 22, streams)))
    n, _ = R.q1_finalize(bytes(R.q1_narrow_fission_run(hn, 1 << 23, streams)))
    if w != ref or n != ref:
        bad += 1
        print("iter", it, "wide ok" if w == ref else "WIDE BAD", "narrow ok" if n == ref else "NARROW BAD", flush=True)
        if n != ref:
            for a, b in zip(n, ref):
                if a != b: print("  narrow", {k: (a[k], b[k]) for k in a if a[k] != b[k]})
        if w != ref:
            for a, b in zip(w, ref):
                if a != b: print("  wide", {k: (a[k], b[k]) for k in a if a[k] != b[k]})
print("bad", bad)
