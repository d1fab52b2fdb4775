"""Map an ncu SASS source page to CUDA source lines (via nvdisasm line info).

usage: python scripts/ncu_lines.py REPORT KERNEL_SUBSTR SOURCE_FILE [N]
"""
import collections, csv, os, re, subprocess, sys, tempfile

rep, kname, srcfile = sys.argv[1], sys.argv[2], sys.argv[3]
N = int(sys.argv[4]) if len(sys.argv) > 4 else 30
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath("paper_conf_ipps_wudwcyc12_b200/libra.so")], cwd=d,
               capture_output=True)
stem = os.path.basename(srcfile).split('.')[0]
cands = sorted(f for f in os.listdir(d) if stem in f and f.endswith(".cubin"))
cub = next((f for f in cands if f == stem + ".sm_100a.cubin"), cands[0])
sass = subprocess.run(["nvdisasm", "--print-line-info", os.path.join(d, cub)], capture_output=True, text=True).stdout
blocks = re.split(r"//-+ \.text\.", sass)
blk = [b for b in blocks if kname in b.split("\n")[0]][0]
cur, insts = None, []
for l in blk.split("\n"):
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    if re.match(r"\s+/\*[0-9a-f]{4,}\*/", l):
        insts.append(cur)
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(src.splitlines()))[2:]
print("instructions: nvdisasm", len(insts), "ncu", len(rows))
inst, stall = collections.Counter(), collections.Counter()
for ln, r in zip(insts, rows):
    inst[ln] += int(r[5])
    stall[ln] += int(r[2])
ti, ts = sum(inst.values()) or 1, sum(stall.values()) or 1
lines = open(srcfile).read().split("\n")
print(f"{'inst%':>6} {'stall%':>6}  line")
for ln, s in stall.most_common(N):
    txt = lines[ln[1] - 1].strip()[:80] if ln and ln[0] == os.path.basename(srcfile) else str(ln)
    print(f"{inst[ln] / ti * 100:6.1f} {s / ts * 100:6.1f}  {ln[1] if ln else '?'}: {txt}")
