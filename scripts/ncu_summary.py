"""Summarise an ncu report: key metrics, stall reasons, hottest SASS lines."""
import csv, subprocess, sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 15
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines()))
h, v = r[0], r[2]
keys = ("gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__grid_size",
        "launch__block_size", "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_bytes.sum", "smsp__inst_executed.sum")
for k, x in zip(h, v):
    if k in keys:
        print(f"{k:60s} {x}")
stalls = [(k, float(x)) for k, x in zip(h, v) if "pcsamp_warps_issue_stalled" in k and not k.endswith("not_issued")
          and x.replace('.', '', 1).isdigit() and float(x) > 0]
tot = sum(s for _, s in stalls)
for k, s in sorted(stalls, key=lambda z: -z[1])[:8]:
    print(f"  stall {k.replace('smsp__pcsamp_warps_issue_stalled_', ''):28s} {s / tot * 100:5.1f}%")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))[2:]
tot = sum(int(x[2]) for x in rows) or 1
top = sorted(range(len(rows)), key=lambda i: -int(rows[i][2]))[:ntop]
for i in top:
    print(f"{i:5d} {int(rows[i][2]) / tot * 100:5.1f}% {rows[i][1].strip()[:58]:58s} <- {rows[i - 1][1].strip()[:40]}")
