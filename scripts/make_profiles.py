"""Summarise ncu captures in gpurun_out/ into tracked profiles/ (per round).

usage: python scripts/make_profiles.py ROUND
Writes profiles/r<ROUND>_<name>.txt (key metrics, stall reasons, hottest SASS),
profiles/r<ROUND>_launches.txt (per-kernel launch list of the bench command)
and updates profiles/ncu_traffic.json (dram bytes per launch, read by bench.py).
"""
import collections
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
RND = sys.argv[1] if len(sys.argv) > 1 else "01"
OUT = os.path.join(ROOT, "profiles")
os.makedirs(OUT, exist_ok=True)

CAPTURES = {  # report -> (summary name, traffic key, command)
    "prof_select": ("select_chain_k2_s05_n28", "select_chain_k2_s0.5_n28",
                    "python scripts/prof_driver.py select 5  (2^28 int32, k=2, s=0.5/stage; select_multi_kernel<1>)"),
    "prof_select_n30": ("select_chain_k2_s05_n30", "select_chain_k2_s0.5_n30",
                        "python scripts/prof_driver.py select 3 30  (2^30 int32, k=2, s=0.5/stage; select_multi_kernel<1>)"),
    "prof_select_s01": ("select_chain_k1_s001_n28", "select_chain_k1_s0.01_n28",
                        "python scripts/prof_driver.py select 5 28 1 0.01  (2^28 int32, k=1, s=0.01; select_multi_kernel<1>)"),
    "prof_select_s09": ("select_chain_k1_s09_n28", "select_chain_k1_s0.9_n28",
                        "python scripts/prof_driver.py select 5 28 1 0.9  (2^28 int32, k=1, s=0.9; select_multi_kernel<1>)"),
    "prof_q1": ("q1_sf10", "q1_sf10", "python scripts/prof_driver.py q1 5  (SF10, 60M rows)"),
    "prof_rows": ("select_rows_k2_s05_n28", "select_rows_k2_s0.5_n28",
                  "python scripts/prof_driver.py rows 5  (2^28 key + 2 int32 fields, k=2, s=0.5/stage)"),
    "prof_q1n": ("q1n_sf10", "q1n_sf10", "python scripts/prof_driver.py q1n 5  (SF10 narrow, 60M rows)"),
    "prof_compact": ("compact_k2_s05_n28", "compact_k2_s0.5_n28",
                     "python scripts/prof_driver.py rows 5  (payload compaction of 3 int32 fields, 2^28 rows, k=2, s=0.5/stage)"),
    "prof_q1_sf100": ("q1_sf100", "q1_sf100", "python scripts/prof_driver.py q1sf100 3  (SF100, 600M rows, one GPU)"),
    "prof_q1n_sf100": ("q1n_sf100", "q1n_sf100", "python scripts/prof_driver.py q1nsf100 3  (SF100 narrow, 600M rows)"),
    "prof_multi": ("select_multi_m2_s05_n28", "select_multi_m2_s0.5_n28",
                   "python scripts/prof_driver.py multi 5 28 2  (2^28 int32, 2 outputs: x<0 | -2^30<x<2^30)"),
    "prof_multi_dense": ("select_multi_m2_s09_n28", "select_multi_m2_s0.9_n28",
                         "python scripts/prof_driver.py multi 5 28 2 0.9  (2^28 int32, 2 outputs keeping ~90% each)"),
    "prof_multi4": ("select_multi_m4_n28", "select_multi_m4_n28",
                    "python scripts/prof_driver.py multi 5 28 4  (2^28 int32, 4 outputs: .5 .5 .25 .25)"),
    "prof_sparse_sel": ("sparse_select_k1_s001_n28", "sparse_select_k1_s0.01_n28",
                        "python scripts/prof_driver.py sparse 5 28 1 0.01  (key pass of the sparse tuple SELECT)"),
    "prof_sparse_ids": ("sparse_ids_k1_s005_n28", "sparse_ids_k1_s0.05_n28",
                        "python scripts/prof_driver.py sparse 5 28 1 0.05  (ids_kernel: the row ids past the n/32 the key pass staged, from the order masks)"),
    "prof_sparse_gather": ("sparse_gather_k1_s001_n28", "sparse_gather_k1_s0.01_n28",
                           "python scripts/prof_driver.py sparse 5 28 1 0.01  (gather_kernel: 3 int32 fields at the ids)"),
}
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
        "launch__shared_mem_per_block_dynamic", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "lts__t_bytes.sum"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    return dict(zip(rows[0], rows[2])), dict(zip(rows[0], rows[1]))


def to_bytes(v, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)
    return float(v.replace(",", "")) * scale


traffic_path = os.path.join(OUT, "ncu_traffic.json")
traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
for rep, (name, tkey, cmd) in CAPTURES.items():
    path = os.path.join(ROOT, "gpurun_out", rep + ".ncu-rep")
    if not os.path.exists(path):
        continue
    vals, units = raw(path)
    lines = [f"# ncu --set full --clock-control none capture, round {RND}", f"# command: {cmd}", ""]
    for k in KEYS:
        if k in vals:
            lines.append(f"{k:60s} {vals[k]:>20s} {units.get(k, '')}")
    rd = to_bytes(vals["dram__bytes_read.sum"], units["dram__bytes_read.sum"])
    wr = to_bytes(vals["dram__bytes_write.sum"], units["dram__bytes_write.sum"])
    traffic[tkey] = rd + wr
    lines.append(f"{'dram bytes read+write per launch':60s} {rd + wr:20.0f} byte")
    stalls = [(k.replace("smsp__pcsamp_warps_issue_stalled_", ""), float(v)) for k, v in vals.items()
              if "pcsamp_warps_issue_stalled" in k and not k.endswith("not_issued")
              and v.replace(".", "", 1).isdigit() and float(v) > 0]
    tot = sum(s for _, s in stalls) or 1
    lines += ["", "warp stall reasons (pc sampling):"]
    lines += [f"  {k:28s} {s / tot * 100:5.1f}%" for k, s in sorted(stalls, key=lambda z: -z[1])[:10]]
    open(os.path.join(OUT, f"r{RND}_{name}.txt"), "w").write("\n".join(lines) + "\n")
    print("wrote", name)
json.dump(traffic, open(traffic_path, "w"), indent=1, sort_keys=True)

lpath = os.path.join(ROOT, "gpurun_out", "launches.csv")
if os.path.exists(lpath):
    rows = [r for r in csv.reader(open(lpath)) if len(r) > 5]
    h = rows[0]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    agg = collections.OrderedDict()
    for r in rows[1:]:
        agg.setdefault(r[ki], []).append(float(r[vi].replace(",", "")))
    total = sum(sum(v) for v in agg.values())
    lines = [f"# round {RND}: ncu --metrics gpu__time_duration.sum --clock-control none -c 400",
             "#   python bench.py --steps 20 --warmup 3 --no-extras   (cold-cache, serialised launches)",
             "# launches  mean_ns  share_of_all  kernel"]
    for k, v in agg.items():
        lines.append(f"{len(v):4d}  {sum(v) / len(v):12.0f}  {sum(v) / total * 100:5.1f}%  {k[:110]}")
    open(os.path.join(OUT, f"r{RND}_launches.txt"), "w").write("\n".join(lines) + "\n")
    print("wrote launches")

# PCIe bytes of the fission paths (ncu application-range replay of scripts/pcie_ranges.py)
ppath = os.path.join(ROOT, "gpurun_out", "pcie.csv")
if os.path.exists(ppath):
    rows = [r for r in csv.reader(open(ppath)) if len(r) > 5]
    h = rows[0]
    ii, mi, ui, vi = h.index("ID"), h.index("Metric Name"), h.index("Metric Unit"), h.index("Metric Value")
    names = ["select_fission_n28", "select_fission_n30", "q1_fission_sf10", "q1n_fission_sf10"]
    per = collections.OrderedDict()
    for r in rows[1:]:
        per.setdefault(int(r[ii]), {})[r[mi]] = (r[vi], r[ui])
    pcie = {}
    lines = [f"# round {RND}: ncu --replay-mode app-range --metrics "
             "pcie__read_bytes.sum,pcie__write_bytes.sum,gpu__time_duration.sum python scripts/pcie_ranges.py",
             "# one range = one synchronous fission call (H2D + kernels + D2H); read = host->device over PCIe",
             "# range                    pcie_read_bytes   pcie_write_bytes   range_ms   read GB/s"]
    for (rid, m), name in zip(sorted(per.items()), names):
        rd = to_bytes(*m["pcie__read_bytes.sum"]) if "pcie__read_bytes.sum" in m else float("nan")
        wr = to_bytes(*m["pcie__write_bytes.sum"]) if "pcie__write_bytes.sum" in m else float("nan")
        t, tu = m.get("gpu__time_duration.sum", ("nan", "ns"))
        ns = float(t.replace(",", "")) * {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6,
                                           "nsecond": 1}.get(tu, 1)
        pcie[name] = {"pcie_read_bytes": rd, "pcie_write_bytes": wr, "range_ns": ns}
        lines.append(f"{name:24s} {rd:17.0f} {wr:18.0f} {ns / 1e6:10.3f} {rd / ns if ns else 0:10.1f}")
    json.dump(pcie, open(os.path.join(OUT, "ncu_pcie.json"), "w"), indent=1, sort_keys=True)
    open(os.path.join(OUT, f"r{RND}_pcie.txt"), "w").write("\n".join(lines) + "\n")
    print("wrote pcie")
