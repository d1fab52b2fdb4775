"""Per-source-line stall samples of one kernel from an ncu report, restricted to
a line range (dev tool): python scripts/ncu_roles.py REP KERNEL_SUBSTR SRC LO HI [N]"""
import collections, csv, os, re, subprocess, sys, tempfile
rep, kname, srcfile, lo, hi = sys.argv[1], sys.argv[2], sys.argv[3], int(sys.argv[4]), int(sys.argv[5])
N = int(sys.argv[6]) if len(sys.argv) > 6 else 25
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath("paper_conf_ipps_wudwcyc12_b200/libra.so")], cwd=d, capture_output=True)
stem = os.path.basename(srcfile).split('.')[0]
sass = subprocess.run(["nvdisasm", "--print-line-info", os.path.join(d, stem + ".sm_100a.cubin")], capture_output=True, text=True).stdout
blk = [b for b in re.split(r"//-+ \.text\.", sass) if kname in b.split("\n")[0]][0]
cur, insts = None, []
stack = []
for l in blk.split("\n"):
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        if "inlined at" in l:
            mm = re.findall(r'inlined at "([^"]+)", line (\d+)', l)
            cur = cur + tuple((os.path.basename(a), int(b)) for a, b in mm)
        continue
    if re.match(r"\s+/\*[0-9a-f]{4,}\*/", l):
        insts.append((cur, l.strip()))
rows = list(csv.reader(subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout.splitlines()))
h = rows[1]
rows = rows[2:]
si = h.index("Warp Stall Sampling (All Samples)")
reasons = [i for i, c in enumerate(h) if c.startswith("stall_") and "Not Issued" not in c]
tot = collections.Counter(); why = collections.defaultdict(collections.Counter); txt = {}
for (ln, sasst), r in zip(insts, rows):
    if not ln:
        continue
    # attribute to the innermost line of this source file within [lo, hi]
    key = None
    for f, n in ([ln[:2]] + list(ln[2:])):
        if f == os.path.basename(srcfile) and lo <= n <= hi:
            key = n
            break
    if key is None:
        continue
    s = int(r[si])
    tot[key] += s
    for i in reasons:
        if int(r[i]):
            why[key][h[i][6:]] += int(r[i])
lines = open(srcfile).read().split("\n")
T = sum(tot.values()) or 1
print(f"lines {lo}-{hi}: {T} samples")
for n, s in tot.most_common(N):
    top = ", ".join(f"{k} {v * 100 // max(1, s)}%" for k, v in why[n].most_common(3))
    print(f"{s * 100 / T:5.1f}%  {n}: {lines[n - 1].strip()[:70]:70s} [{top}]")
