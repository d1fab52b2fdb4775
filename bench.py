#!/usr/bin/env python
"""Benchmark of the fused relational hot path on B200 (one JSON line on rank 0).

Headline (BASELINE.json configs[1]): fused back-to-back SELECTs (k=2, s=0.5
per stage) over 2^28 device-resident int32 rows per GPU; a step is
one fused select_chain kernel (+ at N>1 the NCCL all_gather of the per-rank
counts and the exclusive scan into global output offsets).
`value` = rows/s over all ranks (weak scaling: 2^28 rows per rank).

The same line carries
  roofline      select_fused kernel: algorithmic bytes (4 B in + 4 B per kept
                row out) / mean kernel time vs MEASURED_PEAKS.json hbm_gbs
  e2e           the same chain through ra_fission_run from pinned HOST buffers
                (H2D + D2H inside the timed region), rows/s
  cpu_baseline  the CPU oracle (single thread, as it stands) on the same data
  q1_sf10 / q1_sf100 / select_1m / unfused / sweep  the other BASELINE configs
  clocks        SM clocks and throttle reasons sampled during the timed region

`--impl reference` runs the CPU oracle as the reference arm on the same config.
Launch: python bench.py [--gpus N --steps K --warmup W].  N>1: under torchrun
(WORLD_SIZE must equal N), or without it bench.py re-launches itself as N
ranks through torch.distributed.run.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import ragen  # noqa: E402  (input generator: no method arithmetic)

METRIC = "rows/s (fused SELECT chain k=2 s=0.5, 2^28 int32 rows/GPU, device-resident)"
CHAIN_SEED, Q1_SEED, D1_SEED = 2, 5, 1


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--rows-log2", type=int, default=28)
    ap.add_argument("--k", type=int, default=2)
    ap.add_argument("--sel", type=float, default=0.5)
    ap.add_argument("--no-extras", action="store_true", help="headline only (for ncu runs)")
    ap.add_argument("--sweep", action="store_true", help="selectivity x k sweep, fused vs unfused")
    ap.add_argument("--fission-sweep", action="store_true")
    ap.add_argument("--skip-1g", action="store_true", help="skip the 2^30-row host-resident leg (configs[3])")
    return ap.parse_args()


# ----------------------------------------------------------------- plumbing
class Dist:
    def __init__(self):
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        self.local = int(os.environ.get("LOCAL_RANK", "0"))
        self.pg = None

    def init(self, torch):
        if self.world > 1:
            import torch.distributed as dist
            # RA_BENCH_BACKEND=gloo: exercise the multi-rank code path with several
            # ranks sharing one GPU (functional check only; NCCL needs one GPU per rank)
            backend = os.environ.get("RA_BENCH_BACKEND", "nccl")
            if backend == "nccl":
                if torch.cuda.device_count() < self.world:
                    raise SystemExit(f"bench.py: {self.world} ranks need {self.world} GPUs, "
                                     f"{torch.cuda.device_count()} visible (NCCL: one GPU per rank)")
                dist.init_process_group("nccl", device_id=torch.device("cuda", self.local))
            else:
                dist.init_process_group(backend)
            self.pg = dist

    def device(self, torch) -> int:
        return self.local % torch.cuda.device_count()

    def barrier(self, torch):
        if self.pg:
            self.pg.barrier()
        torch.cuda.synchronize()

    def max(self, torch, v: float) -> float:
        if not self.pg:
            return v
        t = torch.tensor([v], dtype=torch.float64, device="cuda")
        self.pg.all_reduce(t, op=self.pg.ReduceOp.MAX)
        return float(t.item())


class ClockSampler:
    """nvidia-smi-equivalent clocks/throttle sampling (NVML) during a region."""

    REASONS = {
        0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
        0x20: "sw_thermal_slowdown", 0x4: "sw_power_cap", 0x1: "gpu_idle", 0x2: "applications_clocks_setting",
    }

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            self.nv = None
            self.err = str(e)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.nv:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def read_peak():
    """Read-only HBM stream peak measured by scripts/micro/stream_bw.cu (committed
    under profiles/): context for read-dominated kernels, whose fraction of the
    copy (read+write) peak in MEASURED_PEAKS.json can exceed 1."""
    p = os.path.join(ROOT, "profiles", "r01_stream_bw.txt")
    if not os.path.exists(p):
        return None
    best = 0.0
    with open(p) as f:
        for line in f:
            if line.startswith("bulk") and "GB/s" in line:
                best = max(best, float(line.split(":")[1].split()[0]))
    return best or None


def mixed_peak(w: float):
    """Read+write HBM stream peak for a write/read ratio w (scripts/micro/mixed_bw.cu,
    committed under profiles/), linearly interpolated: the ceiling for a SELECT
    writing a fraction w of what it reads."""
    p = os.path.join(ROOT, "profiles", "r01_mixed_bw.txt")
    if not os.path.exists(p):
        return None
    pts = []
    with open(p) as f:
        for line in f:
            if line.startswith("write/read"):
                pts.append((float(line.split(":")[0].split()[-1]), float(line.split("read+write")[1].split()[0])))
    pts.sort()
    for (w0, b0), (w1, b1) in zip(pts, pts[1:]):
        if w0 <= w <= w1:
            return b0 + (b1 - b0) * (w - w0) / (w1 - w0)
    return None


def ncu_pcie(key: str):
    """PCIe bytes (read = host->device) of one fission call from the committed
    ncu application-range capture (scripts/pcie_ranges.py), if any."""
    p = os.path.join(ROOT, "profiles", "ncu_pcie.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f).get(key)
    return None


_PCIE = {}


def pcie_peaks(torch):
    """Pinned host<->device copy bandwidth measured here (the paper's Fig 4(b)
    method): 1 GiB cudaMemcpyAsync each way, best of 3, CUDA events."""
    if _PCIE:
        return _PCIE
    nb, ch = 1 << 30, 1 << 24
    h = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nb, dtype=torch.uint8, device="cuda")
    cur = torch.cuda.current_stream()
    st = [torch.cuda.Stream() for _ in range(3)]

    def chunked(h2d):  # the fission pattern without kernels: 16 MiB chunks round-robin on 3 streams
        for s_ in st:
            s_.wait_stream(cur)
        for c, o in enumerate(range(0, nb, ch)):
            with torch.cuda.stream(st[c % 3]):
                (d[o:o + ch].copy_(h[o:o + ch], non_blocking=True) if h2d else
                 h[o:o + ch].copy_(d[o:o + ch], non_blocking=True))
        for s_ in st:
            cur.wait_stream(s_)

    for name, fns in (("h2d_gbs", (lambda: d.copy_(h, non_blocking=True), lambda: chunked(True))),
                      ("d2h_gbs", (lambda: h.copy_(d, non_blocking=True), lambda: chunked(False)))):
        best = 0.0
        for fn in fns:
            for _ in range(3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                fn()
                e1.record()
                e1.synchronize()
                best = max(best, nb / (e0.elapsed_time(e1) * 1e-3) / 1e9)
        _PCIE[name] = best
    _PCIE["how"] = ("pinned 1 GiB cudaMemcpyAsync, one copy or 16 MiB chunks on 3 streams, best of 3 each, "
                    "measured in this run")
    del h, d
    return _PCIE


def pcie_roofline(torch, h2d_bytes, seconds, ncu_key):
    pk = pcie_peaks(torch)
    ach = h2d_bytes / seconds / 1e9
    cap = ncu_pcie(ncu_key)
    return {"bound": "pcie", "achieved": ach, "peak": pk["h2d_gbs"], "unit": "GB/s", "frac": ach / pk["h2d_gbs"],
            "peak_source": pk["how"], "d2h_peak": pk["d2h_gbs"],
            "traffic": cap["pcie_read_bytes"] if cap else None,
            "traffic_note": "ncu pcie__read_bytes.sum of one call (application-range replay), profiles/ncu_pcie.json"}


def ncu_traffic(key: str):
    """dram bytes per launch from the committed ncu --set full capture, if any."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f).get(key)
    return None


def tuple_traffic(dense: bool, k, s_sel, lg):
    """dram bytes of the tuple SELECT step: key pass + (compaction), from ncu."""
    a = ncu_traffic(f"select_rows_k{k}_s{s_sel}_n{lg}")
    if not dense or a is None:
        return a
    b = ncu_traffic(f"compact_k{k}_s{s_sel}_n{lg}")
    return None if b is None else a + b


class OverlappedExchange:
    """Step i's exchange runs on a side stream reading buffer i & 1 while step
    i+1's kernel runs; the kernel that reuses a buffer (step i+2) waits for the
    exchange that read it.  `join()` before the closing event."""

    def __init__(self, torch, stream, exchange):
        self.torch, self.stream, self.exchange = torch, stream, exchange
        self.side = torch.cuda.Stream(device=stream.device)
        self.kdone = [torch.cuda.Event() for _ in range(2)]
        self.xdone = [None, None]
        self.result = [None, None]

    def after_kernel(self, i, buf):
        t, b = self.torch, i & 1
        self.kdone[b].record(self.stream)
        self.side.wait_event(self.kdone[b])
        with t.cuda.stream(self.side):
            self.result[b] = self.exchange(buf)
            self.xdone[b] = t.cuda.Event()
            self.xdone[b].record(self.side)
        if self.xdone[b ^ 1] is not None:
            self.stream.wait_event(self.xdone[b ^ 1])

    def join(self):
        self.stream.wait_stream(self.side)


def timed(torch, D: Dist, fn, steps: int, warmup: int, kernel_fn=None, join=None):
    """W warm-up steps; then EXACTLY `steps` steps between barrier+sync on both
    sides, CUDA events on the launching (current) stream; max over ranks.
    `join()` (optional) makes the current stream wait for work a step left on
    other streams, before the closing event.  Returns (ms_per_step, mean kernel
    ms or None)."""
    for i in range(warmup):
        fn(i)
    if join:
        join()
    D.barrier(torch)
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)] \
        if kernel_fn else None
    e0.record(s)
    for i in range(steps):
        if kev:
            kev[i][0].record(s)
            kernel_fn(i)
            kev[i][1].record(s)
            fn(i, kernel_done=True)
        else:
            fn(i)
    if join:
        join()
    e1.record(s)
    e1.synchronize()
    D.barrier(torch)
    ms = e0.elapsed_time(e1) / steps
    kms = statistics.mean(a.elapsed_time(b) for a, b in kev) if kev else None
    ms = D.max(torch, ms)
    if kms is not None:
        kms = D.max(torch, kms)
    return ms, kms


# ---------------------------------------------------------------- our arm
def run_ours(args, D: Dist):
    import torch
    D.init(torch)
    torch.cuda.set_device(D.device(torch))
    import paper_conf_ipps_wudwcyc12_b200 as R

    dev = torch.device("cuda", D.device(torch))
    stream = torch.cuda.current_stream()
    sh = int(stream.cuda_stream)
    n = 1 << args.rows_log2
    k, s_sel = args.k, args.sel
    thresholds = ragen.nested_thresholds(s_sel, k)
    preds = [("lt", t) for t in thresholds]
    P = R.make_preds(preds)

    # rank r owns global rows [r*n, (r+1)*n) of one seeded column (weak scaling)
    x = torch.empty(n, dtype=torch.int32, device=dev)
    ragen.int32_column_dev(CHAIN_SEED, x, row0=D.rank * n, stream=sh)
    out = torch.empty(n, dtype=torch.int32, device=dev)
    # step i's count lands in cnts[i & 1]: step i's exchange (side stream) reads
    # it while step i+1's kernel runs; step i+2's kernel waits for that exchange
    cnts = torch.zeros(2, dtype=torch.int64, device=dev)
    ws_bytes = R.ra_select_workspace_bytes(n, k, 1)
    ws = torch.zeros(ws_bytes, dtype=torch.uint8, device=dev)
    from paper_conf_ipps_wudwcyc12_b200 import dist as rdist
    args_chain = [(x.data_ptr(), n, P, k, 1, out.data_ptr(), n, cnts.data_ptr() + 8 * b, ws.data_ptr(), ws_bytes, sh)
                  for b in range(2)]
    side = torch.cuda.Stream(device=dev)
    kdone = [torch.cuda.Event() for _ in range(2)]
    xdone = [None, None]
    gathered = [torch.zeros(D.world, dtype=torch.int64, device=dev) for _ in range(2)]
    offsets = [torch.zeros(D.world, dtype=torch.int64, device=dev) for _ in range(2)]
    totals = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(2)]

    def chain_kernel(i):
        R.ra_select_chain(*args_chain[i & 1])

    def chain_step(i, kernel_done=False):
        if not kernel_done:
            chain_kernel(i)
        if D.pg:  # a9: gather per-rank counts -> exclusive scan -> global offsets,
            b = i & 1  # overlapped with the next step's kernel
            kdone[b].record(stream)
            side.wait_event(kdone[b])
            with torch.cuda.stream(side):
                rdist.exchange_counts(cnts[b:b + 1], counts=gathered[b], offsets=offsets[b], total=totals[b])
                xdone[b] = torch.cuda.Event()
                xdone[b].record(side)
            if xdone[b ^ 1] is not None:  # the next kernel reuses the buffer step i-1's exchange read
                stream.wait_event(xdone[b ^ 1])

    def join():
        if D.pg:
            stream.wait_stream(side)

    torch.cuda.synchronize()
    launches0 = R.ra_kernel_launches()
    with ClockSampler(D.device(torch)) as clk:
        # at N=1 a step is exactly one kernel launch, back to back on one stream
        # (programmatic dependent launch overlaps each launch with the previous
        # kernel's tail; an event between them would break that), so the
        # kernel's mean duration is the timed region / K; at N>1 each kernel is
        # bracketed by its own events
        ms, kms = timed(torch, D, chain_step, args.steps, args.warmup,
                        kernel_fn=chain_kernel if D.pg else None, join=join)
        kms = ms if kms is None else kms
    launches = R.ra_kernel_launches() - launches0 - args.warmup
    last = (args.steps - 1) & 1
    cnt = cnts[last:last + 1]
    kept = int(cnt.item())
    if D.pg:  # the exchange's result: this rank's count, offset = counts of lower ranks, total
        g = [int(v) for v in gathered[last].tolist()]
        assert g[D.rank] == kept
        assert int(offsets[last][D.rank].item()) == sum(g[:D.rank]) and int(totals[last].item()) == sum(g)
    value = D.world * n / (ms * 1e-3)
    peak, peak_src = peaks()
    alg_bytes = 4 * n + 4 * kept
    achieved = alg_bytes / (kms * 1e-3) / 1e9
    res = {
        "metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": D.world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "int32", "data": "synthetic (seeded uniform int32, ragen)",
        "config": {"workload": f"configs[1]: fused {k}x SELECT, s={s_sel}/stage, 2^{args.rows_log2} int32 rows/GPU, device-resident",
                   "rows_per_gpu": n, "k": k, "sel_per_stage": s_sel, "kept_per_gpu": kept,
                   "l2": "inputs > L2 (1 GiB column per step vs 126 MB L2), no flush needed",
                   "parallelism": f"row-range shards x{D.world}, NCCL all_gather of counts"},
        "gpu_launches": launches,
        "roofline": {"kernel": "select_multi_kernel<M=1> (the fused chain)", "bound": "hbm", "achieved": achieved,
                     "peak": peak, "peak_source": peak_src, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": ncu_traffic(f"select_chain_k{k}_s{s_sel}_n{args.rows_log2}"),
                     "algorithmic_bytes_per_launch": alg_bytes, "kernel_ms": kms,
                     "mixed_stream_peak": mixed_peak(kept / n),
                     "frac_of_mixed_stream_peak": (achieved / mixed_peak(kept / n)) if mixed_peak(kept / n) else None},
        "clocks": clk.summary(),
    }
    if not args.no_extras:
        res.update(extras(args, D, torch, R, x, preds, kept, ms))
    if D.rank == 0:
        print(json.dumps(res), flush=True)


def extras(args, D, torch, R, x, preds, kept, chain_ms):
    """Other BASELINE configs + e2e + CPU baseline, same timing rules."""
    from paper_conf_ipps_wudwcyc12_b200 import dist as rdist
    s_sel = args.sel
    dev = x.device
    sh = int(torch.cuda.current_stream().cuda_stream)
    n = x.numel()
    k = len(preds)
    peak, _ = peaks()
    ex = {}

    # --- unfused composition of the same chain (the paper's "without round trip")
    if k > 1:
        uo = torch.empty(n, dtype=torch.int32, device=dev)
        uc = torch.zeros(1, dtype=torch.int64, device=dev)
        uws_b = R.ra_select_workspace_bytes(n, k, 0)
        uws = torch.zeros(uws_b, dtype=torch.uint8, device=dev)
        P = R.make_preds(preds)
        a = (x.data_ptr(), n, P, k, 0, uo.data_ptr(), n, uc.data_ptr(), uws.data_ptr(), uws_b, sh)
        ums, _ = timed(torch, D, lambda i, kernel_done=False: R.ra_select_chain(*a), 20, 3)
        assert int(uc.item()) == kept
        ex["unfused"] = {"rows_per_s": D.world * n / (ums * 1e-3), "ms_per_step": ums,
                         "fused_over_unfused": ums / chain_ms, "launches_per_step": k}
        del uo, uws

    # --- library yardstick: the same chain as PyTorch ops
    # (elementwise compares -> mask -> torch.masked_select); not our path
    def torch_chain(i=0, kernel_done=False):
        m = x < preds[0][1]
        for _, t in preds[1:]:
            m &= x < t
        return torch.masked_select(x, m)
    assert torch_chain().numel() == kept
    tms_, _ = timed(torch, D, torch_chain, 10, 3)
    ex["yardstick_torch_masked_select"] = {"ms_per_step": tms_, "ours_speedup": tms_ / chain_ms,
                                           "ops": "x < T_j (k compares, &=) then torch.masked_select"}

    # --- e2e: same chain from pinned host memory through ra_fission_run
    if True:  # every rank streams its own shard from pinned host memory
        h_in = torch.empty(n, dtype=torch.int32, pin_memory=True)
        h_in.copy_(x.cpu())
        h_out = torch.empty(n, dtype=torch.int32, pin_memory=True)
        chunk = 1 << 24
        streams = [torch.cuda.Stream() for _ in range(3)]
        h_counts = torch.zeros((n + chunk - 1) // chunk, dtype=torch.int64, pin_memory=True)
        def fission_ms(chunk, S, fused, reps=3):
            st = streams[:S]
            R.fission_run(h_in, preds, chunk, st, fused=fused, h_out=h_out, h_chunk_counts=h_counts)
            # synchronous host API: bracket it with events on the current stream (device clock)
            ms, _ = timed(torch, D, lambda i, kernel_done=False: R.fission_run(
                h_in, preds, chunk, st, fused=fused, h_out=h_out, h_chunk_counts=h_counts), reps, 1)
            return ms

        dt = fission_ms(chunk, 3, True) * 1e-3
        _, c = R.fission_run(h_in, preds, chunk, streams, h_out=h_out, h_chunk_counts=h_counts)
        assert c == kept
        ex["e2e"] = {"value": D.world * n / dt, "unit": "rows/s", "h2d_bytes_per_step": 4 * n,
                     "d2h_bytes_per_step": 4 * c + 8 * ((n + chunk - 1) // chunk), "ms_per_step": dt * 1e3,
                     "path": "ra_fission_run: pinned host in/out, chunk 2^24 rows, 3 streams (fusion+fission)",
                     "pcie_h2d_gbs": 4 * n / dt / 1e9,
                     "roofline": pcie_roofline(torch, 4 * n, dt, "select_fission_n28")}
        # d4: the paper's Fig 16 modes on the same host-resident chain
        modes = {"serial": (n, 1, False), "fusion_only": (n, 1, True),
                 "fission_only": (chunk, 3, False), "fusion_fission": (chunk, 3, True)}
        ex["fission_modes"] = {m: {"ms_per_step": fission_ms(*cfg), "chunk_rows": cfg[0], "streams": cfg[1],
                                   "fused": cfg[2]} for m, cfg in modes.items()}
        # the paper's "with round trip" (Fig 8): each SELECT copies its
        # input to the GPU and its result back; the next SELECT starts from the host
        if k > 1:
            h_mid = torch.empty(n, dtype=torch.int32, pin_memory=True)
            bufs = [h_out, h_mid]

            def round_trip(i=0, kernel_done=False):
                src, m = h_in, n
                for j, pj in enumerate(preds):
                    dst = bufs[j & 1]
                    _, m = R.fission_run(src[:m], [pj], m, streams[:1], h_out=dst, h_chunk_counts=h_counts)
                    src = dst
                return m

            assert round_trip() == kept
            rms, _ = timed(torch, D, round_trip, 3, 1)
            ex["fission_modes"]["with_round_trip"] = {"ms_per_step": rms, "chunk_rows": n, "streams": 1,
                                                      "fused": False, "selects": k}
            del h_mid
        for v in ex["fission_modes"].values():
            v["rows_per_s"] = D.world * n / (v["ms_per_step"] * 1e-3)
        del h_in, h_out, h_counts

    # --- configs[3]: host-resident chain on 2^30 rows with fission (4 GiB pinned in)
    if D.world == 1 and not args.skip_1g:  # one rank (its timed() has collectives)
        n3 = 1 << 30
        h3 = torch.empty(n3, dtype=torch.int32, pin_memory=True)
        ragen.int32_column(4, n3, out=h3.numpy())
        o3 = torch.empty(n3, dtype=torch.int32, pin_memory=True)
        st3 = [torch.cuda.Stream() for _ in range(3)]
        cc3 = torch.zeros(n3 >> 24, dtype=torch.int64, pin_memory=True)
        _, k3 = R.fission_run(h3, preds, 1 << 24, st3, h_out=o3, h_chunk_counts=cc3)
        # full-size consistency: the device-resident fused chain on the same rows
        d3 = h3.cuda()
        dout, dcnt = R.select_chain(d3, preds)
        assert int(dcnt.item()) == k3, "fission and device-resident counts differ"
        idx = torch.randint(0, k3, (1 << 16,), generator=torch.Generator().manual_seed(7))
        assert torch.equal(dout[idx.cuda()].cpu(), o3[idx]), "fission output differs from the device result"
        del d3, dout
        f3ms, _ = timed(torch, D, lambda i, kernel_done=False: R.fission_run(
            h3, preds, 1 << 24, st3, h_out=o3, h_chunk_counts=cc3), 3, 1)
        ex["fission_1g"] = {"workload": "configs[3]: host-resident 2^30 int32 rows (seed 4), k=2 s=.5/stage, "
                                        "chunk 2^24, 3 streams, fusion+fission",
                            "rows": n3, "kept": k3, "ms_per_step": f3ms, "rows_per_s": n3 / (f3ms * 1e-3),
                            "checked": "count + 65536 sampled outputs equal the device-resident fused chain",
                            "h2d_bytes_per_step": 4 * n3, "d2h_bytes_per_step": 4 * k3 + 8 * (n3 >> 24),
                            "pcie_h2d_gbs": 4 * n3 / (f3ms * 1e-3) / 1e9,
                            "roofline": pcie_roofline(torch, 4 * n3, f3ms * 1e-3, "select_fission_n30")}
        del h3, o3

    # --- d5 shape for SELECT: 2^30 device-resident rows split across the ranks
    # (strong scaling), fused k-chain + the count exchange
    nb = (1 << 30) // D.world
    xb = torch.empty(nb, dtype=torch.int32, device=dev)
    ragen.int32_column_dev(CHAIN_SEED + 200, xb, row0=D.rank * nb, stream=sh)
    ob = torch.empty(nb, dtype=torch.int32, device=dev)
    cb = torch.zeros(1, dtype=torch.int64, device=dev)
    gb, ofb, tob = (torch.zeros(m, dtype=torch.int64, device=dev) for m in (D.world, D.world, 1))
    wsb_b = R.ra_select_workspace_bytes(nb, k, 1)
    wsb = torch.zeros(wsb_b, dtype=torch.uint8, device=dev)
    Pb = R.make_preds(preds)
    ab = (xb.data_ptr(), nb, Pb, k, 1, ob.data_ptr(), nb, cb.data_ptr(), wsb.data_ptr(), wsb_b, sh)

    def big_step(i, kernel_done=False):
        if not kernel_done:
            R.ra_select_chain(*ab)
        if D.pg:
            rdist.exchange_counts(cb, counts=gb, offsets=ofb, total=tob)

    bms, bkms = timed(torch, D, big_step, 20, 3, kernel_fn=lambda i: R.ra_select_chain(*ab))
    bk = int(cb.item())
    bach = (4 * nb + 4 * bk) / (bkms * 1e-3) / 1e9
    ex["select_1g_device"] = {"workload": f"2^30 int32 rows device-resident, split over {D.world} rank(s), k={k}, "
                                          f"s={s_sel}/stage (SURVEY d5 shape)",
                              "rows": 1 << 30, "rows_per_s": (1 << 30) / (bms * 1e-3), "ms_per_step": bms,
                              "kernel_ms": bkms, "scaling": "strong",
                              "roofline": {"kernel": "select_multi_kernel<M=1>", "bound": "hbm", "achieved": bach,
                                           "peak": peak, "unit": "GB/s", "frac": bach / peak,
                                           "algorithmic_bytes_per_launch": 4 * nb + 4 * bk,
                                           "traffic": ncu_traffic(f"select_chain_k{k}_s{s_sel}_n{nb.bit_length() - 1}")
                                           if nb & (nb - 1) == 0 else None}}
    del xb, ob, wsb

    # --- f2: several SELECTs filtering the same input (Fig 2(c)): one fused pass
    # (select_multi_kernel<M>, one input read) vs the M SELECT passes run one
    # after the other (M input reads); M = 2 (the bench pair) and M = 4
    def multi_leg(chains, key):
        M = len(chains)
        mo = [torch.empty(n, dtype=torch.int32, device=dev) for _ in range(M)]
        mc = torch.zeros(M, dtype=torch.int64, device=dev)
        mws_b = R.ra_select_multi_workspace_bytes(n)
        mws = torch.zeros(mws_b, dtype=torch.uint8, device=dev)
        keepP = [R.make_preds(c) for c in chains]
        mch = (ctypes.c_void_p * M)(*[ctypes.addressof(p_) for p_ in keepP])
        mks = (ctypes.c_int * M)(*[len(c) for c in chains])
        mop = (ctypes.c_void_p * M)(*[o.data_ptr() for o in mo])
        mcap = (ctypes.c_int64 * M)(*([n] * M))
        mcp = (ctypes.c_void_p * M)(*[mc.data_ptr() + 8 * o for o in range(M)])
        am = (x.data_ptr(), n, mch, mks, M, mop, mcap, mcp, mws.data_ptr(), mws_b, sh)
        mms, _ = timed(torch, D, lambda i, kernel_done=False: R.ra_select_multi(*am), 20, 3)
        cs = [int(v) for v in mc.cpu().tolist()]
        sws_b = R.ra_select_workspace_bytes(n, RA_MAX_PREDS, 1)
        sws = torch.zeros(sws_b, dtype=torch.uint8, device=dev)
        sep = [(x.data_ptr(), n, keepP[o], len(chains[o]), 1, mo[o].data_ptr(), n, mc.data_ptr() + 8 * o,
                sws.data_ptr(), sws_b, sh) for o in range(M)]

        def separate(i=0, kernel_done=False):
            for a in sep:
                R.ra_select_chain(*a)
        sms, _ = timed(torch, D, separate, 20, 3)
        assert [int(v) for v in mc.cpu().tolist()] == cs
        malg = 4 * n + 4 * sum(cs)
        mach = malg / (mms * 1e-3) / 1e9
        return {"outputs": M, "chains": [[list(p_) for p_ in c] for c in chains], "kept": cs,
                "rows_per_s": D.world * n / (mms * 1e-3), "ms_per_step": mms,
                "separate_selects_ms": sms, "fused_over_separate": sms / mms,
                "bytes_ratio": (4 * M * n + 4 * sum(cs)) / malg,
                "roofline": {"kernel": f"select_multi_kernel<M={M}>", "bound": "hbm", "achieved": mach,
                             "peak": peak, "unit": "GB/s", "frac": mach / peak, "algorithmic_bytes_per_launch": malg,
                             "traffic": ncu_traffic(key),
                             "mixed_stream_peak": mixed_peak(sum(cs) / n),
                             "frac_of_mixed_stream_peak": mach / mixed_peak(sum(cs) / n) if mixed_peak(sum(cs) / n)
                             else None}}

    from paper_conf_ipps_wudwcyc12_b200 import RA_MAX_PREDS
    ex["select_multi"] = multi_leg([[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)]], "select_multi_m2_s0.5_n28")
    ex["select_multi"]["m4"] = multi_leg([[("lt", 0)], [("gt", -(2**30)), ("lt", 2**30)], [("ge", 2**30)],
                                          [("lt", -(2**30))]], "select_multi_m4_n28")

    # --- f3: tuple SELECT (Table I) on the same key column + two int32 fields,
    # the same chain; outputs the key and both fields of the selected rows
    f1 = torch.empty(n, dtype=torch.int32, device=dev)
    f2 = torch.empty(n, dtype=torch.int32, device=dev)
    ragen.int32_column_dev(CHAIN_SEED + 100, f1, stream=sh)
    ragen.int32_column_dev(CHAIN_SEED + 101, f2, stream=sh)
    outs = [torch.empty(n, dtype=torch.int32, device=dev) for _ in range(3)]
    pl = (R.ra_payload * 3)()
    for j, (c, o) in enumerate(zip((x, f1, f2), outs)):
        pl[j].col, pl[j].out, pl[j].elem_bytes = c.data_ptr(), o.data_ptr(), 4
    tc = torch.zeros(1, dtype=torch.int64, device=dev)
    tws_b = R.ra_select_rows_workspace_bytes(n, k)
    tws = torch.zeros(tws_b, dtype=torch.uint8, device=dev)
    PT = R.make_preds(preds)
    at = (x.data_ptr(), n, PT, k, 0, pl, 3, n, tc.data_ptr(), tws.data_ptr(), tws_b, sh)
    tms, _ = timed(torch, D, lambda i, kernel_done=False: R.ra_select_rows(*at), 20, 3)
    tkms = tms  # select + gather/compaction kernels back to back (the whole step)
    tk = int(tc.item())
    assert tk == kept
    dense = tk * 32 > n  # the device's choice (ra_select_rows, 4-byte fields)
    if dense:  # key read, order masks (n/8) written + read, 3 columns streamed, 3 fields written
        talg = 4 * n + 2 * (n // 8) + 3 * 4 * n + 3 * 4 * tk
        kname = "select_fused_kernel<ROWS> + compact_kernel"
    else:  # key read, ids written + read back, 3 fields gathered + written
        talg = 4 * n + 2 * 4 * tk + 3 * 4 * tk + 3 * 4 * tk
        kname = "select_fused_kernel<ROWS> + gather_kernel"
    tach = talg / (tkms * 1e-3) / 1e9
    ex["tuple_select"] = {"rows_per_s": D.world * n / (tms * 1e-3), "ms_per_step": tms, "kernel_ms": tkms,
                          "fields": 3, "kept": tk, "payload_path": "compaction" if dense else "gather",
                          "roofline": {"kernel": kname, "bound": "hbm", "achieved": tach,
                                       "peak": peak, "unit": "GB/s", "frac": tach / peak,
                                       "algorithmic_bytes_per_launch": talg,
                                       "traffic": tuple_traffic(dense, k, s_sel, n.bit_length() - 1)}}
    del f1, f2, outs, tws

    # --- configs[0]: single SELECT on 2^20 rows, 50% (latency-bound, L2-resident)
    n1 = 1 << 20
    x1 = torch.empty(n1, dtype=torch.int32, device=dev)
    ragen.int32_column_dev(D1_SEED, x1, stream=sh)
    o1 = torch.empty(n1, dtype=torch.int32, device=dev)
    c1 = torch.zeros(1, dtype=torch.int64, device=dev)
    ws1_b = R.ra_select_workspace_bytes(n1, 1, 1)
    ws1 = torch.zeros(ws1_b, dtype=torch.uint8, device=dev)
    P1 = R.make_preds([("lt", 0)])
    a1 = (x1.data_ptr(), n1, P1, 1, 1, o1.data_ptr(), n1, c1.data_ptr(), ws1.data_ptr(), ws1_b, sh)
    ms1, _ = timed(torch, D, lambda i, kernel_done=False: R.ra_select_chain(*a1), 200, 10)
    ex["select_1m"] = {"us_per_call": ms1 * 1e3, "rows_per_s": n1 / (ms1 * 1e-3), "kept": int(c1.item()),
                       "note": "configs[0]; 6 MiB L2-resident; back-to-back C-ABI calls from Python (the "
                               "ctypes call itself takes ~6-8 us on the host, so this can be host-bound); "
                               "graph_us_per_call = the same calls replayed from a CUDA graph (device time)"}
    try:  # d1: CUDA-graph replay of 100 captured C-ABI calls (launch latency off the host)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            shc = int(torch.cuda.current_stream().cuda_stream)
            for _ in range(100):
                R.ra_select_chain(*a1[:-1], shc)
        gms, _ = timed(torch, D, lambda i, kernel_done=False: g.replay(), 10, 3)
        ex["select_1m"]["graph_us_per_call"] = gms * 1e3 / 100
        assert int(c1.item()) == ex["select_1m"]["kept"]
        del g
    except Exception as e:  # noqa: BLE001 — report, do not lose the rest of the line
        ex["select_1m"]["graph_error"] = repr(e)[:200]

    # --- configs[2]: Q1 SF10 device-resident (N=1 only) and configs[4] SF100 sharded
    def q1_bench(sf, shard):
        N = ragen.rows_for_sf(sf)
        from paper_conf_ipps_wudwcyc12_b200 import dist as rdist
        lo, hi = rdist.shard_range(N, D.rank, D.world) if shard else (0, N)
        m = hi - lo
        cols = {name: torch.empty(m, dtype=getattr(torch, np.dtype(dt).name), device=dev)
                for name, dt in ragen.LINEITEM_COLUMNS}
        ragen.lineitem_dev(Q1_SEED, ragen.parts_for_sf(sf), cols, row0=lo, stream=sh)
        # step i's partial lands in part[i & 1]; at N > 1 its all_gather (the a9
        # exchange) overlaps step i+1's kernel (OverlappedExchange)
        part = [torch.zeros(ctypes.sizeof(R.ra_q1_partial), dtype=torch.uint8, device=dev) for _ in range(2)]
        wsq_b = R.ra_q1_workspace_bytes(m)
        wsq = torch.zeros(wsq_b, dtype=torch.uint8, device=dev)
        li = R.lineitem_struct(cols)
        xq = OverlappedExchange(torch, torch.cuda.current_stream(), rdist.gather_partials)
        exch = D.pg is not None and shard

        def kern(i):
            R.ra_q1(li, m, R.Q1_CUTOFF_DELTA90, part[i & 1].data_ptr(), wsq.data_ptr(), wsq_b, sh)

        def step(i, kernel_done=False):
            if not kernel_done:
                kern(i)
            if exch:
                xq.after_kernel(i, part[i & 1])

        # without an exchange a step is one kernel launch, timed back to back (see run_ours)
        qms, qkms = timed(torch, D, step, 50, 5, kernel_fn=kern if exch else None, join=xq.join if exch else None)
        qkms = qms if qkms is None else qkms
        last = (50 - 1) & 1
        raw = (xq.result[last] if exch else part[last]).cpu().numpy().tobytes()
        rows, rc = R.q1_finalize(raw)
        ach = 38 * m / (qkms * 1e-3) / 1e9
        res = {"rows": N, "rows_per_s": (N if shard else m) / (qms * 1e-3), "ms_per_step": qms,
               "kernel_ms": qkms, "groups": len(rows), "finalize_rc": rc,
               "roofline": {"kernel": "q1_tma_kernel", "bound": "hbm", "achieved": ach, "peak": peak,
                            "unit": "GB/s", "frac": ach / peak, "algorithmic_bytes_per_launch": 38 * m,
                            "traffic": ncu_traffic(f"q1_sf{int(sf)}"), "read_stream_peak": read_peak(),
                            "frac_of_read_stream_peak": ach / read_peak() if read_peak() else None}}

        # f4: the same rows re-encoded narrow (11 B/row), same partial / finalize
        enc, est = R.q1_encode(cols, stream=torch.cuda.current_stream())
        del cols
        assert int(est.item()) == 0
        hn = R.ra_lineitem_narrow(*[enc[name].data_ptr() for name, _ in R.NARROW_COLUMNS])

        def nkern(i):
            R.ra_q1_narrow(hn, m, R.Q1_CUTOFF_DELTA90, part[i & 1].data_ptr(), wsq.data_ptr(), wsq_b, sh)

        def nstep(i, kernel_done=False):
            if not kernel_done:
                nkern(i)
            if exch:
                xq.after_kernel(i, part[i & 1])

        nms, nkms = timed(torch, D, nstep, 50, 5, kernel_fn=nkern if exch else None, join=xq.join if exch else None)
        nkms = nms if nkms is None else nkms
        nrows, nrc = R.q1_finalize((xq.result[last] if exch else part[last]).cpu().numpy().tobytes())
        assert nrows == rows, "narrow and wide Q1 disagree"
        nach = 11 * m / (nkms * 1e-3) / 1e9
        res["narrow"] = {"rows_per_s": (N if shard else m) / (nms * 1e-3), "ms_per_step": nms, "kernel_ms": nkms,
                         "bytes_per_row": 11, "same_result_as_wide": True,
                         "roofline": {"kernel": "q1n_kernel", "bound": "hbm", "achieved": nach, "peak": peak,
                                      "unit": "GB/s", "frac": nach / peak, "algorithmic_bytes_per_launch": 11 * m,
                                      "traffic": ncu_traffic(f"q1n_sf{int(sf)}"),
                                      "note": "issue/shared-memory bound (per-row group-record update), see DESIGN.md"}}
        del enc
        return res

    if D.world == 1:
        ex["q1_sf10"] = q1_bench(10, False)
        ex["q1_sf10"]["e2e"] = q1_e2e(args, D, torch, R, 10)
        ex["q1_sf10"]["cpu_baseline"] = ex["q1_sf10"]["e2e"].pop("cpu_baseline")
    ex["q1_sf100"] = q1_bench(100, True)
    ex["q1_sf100"]["scaling"] = "strong (600M rows split over ranks)"

    # --- CPU baseline: the oracle as it stands, rank 0, N=1 only
    if D.world == 1 and D.rank == 0:
        ex["cpu_baseline"] = cpu_baseline(x, preds, n)
    return ex


def q1_e2e(args, D, torch, R, sf):
    """Q1 from pinned host columns through ra_q1_fission_run (f1): H2D of the
    38 B/row inside the timed region, the 400-B partial read back every step."""
    N = ragen.rows_for_sf(sf)
    cols = ragen.lineitem(Q1_SEED, N, ragen.parts_for_sf(sf))
    h = {k: torch.from_numpy(v).pin_memory() for k, v in cols.items()}
    streams = [torch.cuda.Stream() for _ in range(3)]
    chunk = 1 << 22
    part = R.q1_fission_run(h, chunk, streams)
    ms, _ = timed(torch, D, lambda i, kernel_done=False: R.q1_fission_run(h, chunk, streams), 3, 1)
    rows, rc = R.q1_finalize(bytes(part))
    cpu = cpu_baseline_q1(cols, R.Q1_CUTOFF_DELTA90, rows) if D.rank == 0 else None
    del cols
    res = {"value": N / (ms * 1e-3), "unit": "rows/s", "h2d_bytes_per_step": 38 * N,
           "d2h_bytes_per_step": 3 * ctypes.sizeof(R.ra_q1_partial), "ms_per_step": ms,
           "pcie_h2d_gbs": 38 * N / (ms * 1e-3) / 1e9, "groups": len(rows), "finalize_rc": rc,
           "roofline": pcie_roofline(torch, 38 * N, ms * 1e-3, "q1_fission_sf10"),
           "path": "ra_q1_fission_run: pinned host columns, chunk 2^22 rows, 3 streams"}
    # f1 x f4: the same table held narrow (11 B/row) in pinned host memory
    dcols = {k: v.cuda() for k, v in h.items()}
    dref, _ = R.q1_finalize(bytes(R.q1(dcols).cpu().numpy().tobytes()))  # device-resident check value
    del h
    enc, st = R.q1_encode(dcols)
    del dcols
    assert int(st.item()) == 0
    hn = {k: v.cpu().pin_memory() for k, v in enc.items()}
    del enc
    chunk_n = 1 << 23
    npart = R.q1_narrow_fission_run(hn, chunk_n, streams)
    nms, _ = timed(torch, D, lambda i, kernel_done=False: R.q1_narrow_fission_run(hn, chunk_n, streams), 3, 1)
    nrows, nrc = R.q1_finalize(bytes(npart))
    if nrows != rows or rows != dref:  # a bit-exact system prints no number next to a mismatch
        raise SystemExit(f"q1_e2e parity FAILED: wide == device {rows == dref}, narrow == device {nrows == dref}")
    res["check"] = "wide and narrow fission results equal the device-resident query"
    res["cpu_baseline"] = cpu
    res["narrow"] = {"value": N / (nms * 1e-3), "unit": "rows/s", "h2d_bytes_per_step": 11 * N,
                     "d2h_bytes_per_step": 3 * ctypes.sizeof(R.ra_q1_partial), "ms_per_step": nms,
                     "pcie_h2d_gbs": 11 * N / (nms * 1e-3) / 1e9,
                     "roofline": pcie_roofline(torch, 11 * N, nms * 1e-3, "q1n_fission_sf10"),
                     "path": "ra_q1_narrow_fission_run: pinned host narrow columns, chunk 2^23 rows, 3 streams"}
    del hn
    return res


def oracle_select_threads(xh, preds, T):
    """The oracle (as it stands) on T host threads: contiguous row ranges, each
    an oracle_select call (ctypes releases the GIL), concatenated in order
    (chunked SELECT == SELECT)."""
    import oracle  # test infrastructure: only bench.py's CPU legs may use it
    from concurrent.futures import ThreadPoolExecutor
    if T <= 1:
        return oracle.select(xh, preds)
    cuts = [len(xh) * r // T for r in range(T + 1)]
    with ThreadPoolExecutor(T) as ex:
        parts = list(ex.map(lambda r: oracle.select(xh[cuts[r]:cuts[r + 1]], preds), range(T)))
    return np.concatenate(parts)


def host_threads() -> int:
    return len(os.sched_getaffinity(0))


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def median_of_3(fn):
    """(median wall seconds of 3 runs, last result)."""
    ts, r = [], None
    for _ in range(3):
        t0 = time.perf_counter()
        r = fn()
        ts.append(time.perf_counter() - t0)
    return statistics.median(ts), r


def cpu_baseline(x, preds, n):
    """The SELECT oracle as it stands: 1 thread and T threads, median of 3."""
    T = host_threads()
    s1 = min(n, 1 << 26)
    x1 = x[:s1].cpu().numpy()
    t1, o1 = median_of_3(lambda: oracle_select_threads(x1, preds, 1))
    sT = min(n, 1 << 28)
    xT = x[:sT].cpu().numpy()
    tT, oT = median_of_3(lambda: oracle_select_threads(xT, preds, T))
    return {"value": sT / tT, "unit": "rows/s", "cores": T, "kind": "oracle", "cpu": cpu_model(),
            "sample": f"first 2^{sT.bit_length() - 1} rows of the same column, oracle_select (C, -O2) on {T} "
                      f"threads over contiguous row ranges, outputs concatenated; median of 3",
            "kept": int(oT.size), "single_thread": {"value": s1 / t1, "cores": 1, "kept": int(o1.size),
                                                    "sample": f"first 2^{s1.bit_length() - 1} rows, 1 thread, "
                                                              f"median of 3"}}


def oracle_q1_threads(cols, T, cutoff):
    """oracle_q1 (as it stands) on T host threads over contiguous row ranges;
    the per-range exact sums are added per group (partition additivity) and
    the AVGs recomputed as one division of exact operands (C12)."""
    import oracle  # test infrastructure: only bench.py's CPU legs may use it
    from concurrent.futures import ThreadPoolExecutor
    n = int(cols["shipdate"].size)
    if T <= 1:
        return oracle.q1(cols, cutoff)[0]
    cuts = [n * r // T for r in range(T + 1)]
    with ThreadPoolExecutor(T) as ex:
        parts = list(ex.map(lambda r: oracle.q1({k: v[cuts[r]:cuts[r + 1]] for k, v in cols.items()}, cutoff)[0],
                            range(T)))
    acc = {}
    sums = ("count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc")
    for rows in parts:
        for r in rows:
            a = acc.setdefault((r["rf_byte"], r["ls_byte"]), dict(r, **{k: 0 for k in sums}))
            for k in sums:
                a[k] += r[k]
    out = [acc[key] for key in sorted(acc)]
    for a in out:
        den = float(a["count_order"] * 100)
        a["avg_qty"], a["avg_price"], a["avg_disc"] = (float(a["sum_qty"]) / den, float(a["sum_base_price"]) / den,
                                                       float(a["sum_disc"]) / den)
    return out


def cpu_baseline_q1(cols, cutoff, gpu_rows):
    """The Q1 oracle as it stands on the SF10 table: 1 thread and T threads,
    median of 3; its result is checked against the GPU's."""
    T = host_threads()
    n = int(cols["shipdate"].size)
    t1, r1 = median_of_3(lambda: oracle_q1_threads(cols, 1, cutoff))
    tT, rT = median_of_3(lambda: oracle_q1_threads(cols, T, cutoff))
    keys = ("count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc",
            "avg_qty", "avg_price", "avg_disc")
    same = all(len(r) == len(gpu_rows) and all(a[k] == b[k] for a, b in zip(r, gpu_rows) for k in keys)
               for r in (r1, rT))
    if not same:
        raise SystemExit("q1 cpu_baseline: the oracle's result differs from the GPU's")
    return {"value": n / tT, "unit": "rows/s", "cores": T, "kind": "oracle", "cpu": cpu_model(),
            "sample": f"the whole SF10 table ({n} rows, host-resident), oracle_q1 (C, -O2, exact 128-bit sums) on {T} "
                      "threads over contiguous row ranges, group sums added exactly; median of 3",
            "same_result_as_gpu": True,
            "single_thread": {"value": n / t1, "cores": 1, "sample": "the whole SF10 table, 1 thread, median of 3"}}


# ---------------------------------------------------------- reference arm
def run_reference(args, D: Dist):
    """The CPU oracle as the reference arm, same config/metric/unit."""
    if D.rank != 0:
        return
    n = 1 << args.rows_log2
    sample = min(n, 1 << 26)
    T = host_threads()
    x = ragen.int32_column(CHAIN_SEED, sample)
    preds = [("lt", t) for t in ragen.nested_thresholds(args.sel, args.k)]
    for _ in range(max(1, args.warmup)):
        oracle_select_threads(x, preds, T)
    steps = max(1, min(args.steps, 20))
    t0 = time.perf_counter()
    for _ in range(steps):
        out = oracle_select_threads(x, preds, T)
    dt = (time.perf_counter() - t0) / steps
    v = sample / dt
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "rows/s", "n_gpus": args.gpus,
        "steps": steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic (seeded uniform int32, ragen)",
        "config": {"workload": f"configs[1]: fused {args.k}x SELECT, s={args.sel}/stage, 2^{args.rows_log2} int32 rows; "
                               f"oracle step = bounded sample of 2^26 rows", "kept": int(out.size)},
        "cpu_baseline": {"value": v, "unit": "rows/s", "cores": T, "kind": "oracle", "cpu": cpu_model(),
                         "sample": f"2^26 rows of the configs[1] column per step (plain C oracle on {T} threads "
                                   f"over contiguous row ranges, outputs concatenated)"},
        "e2e": {"value": v, "unit": "rows/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def _free_port() -> int:
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def launch_ranks(args) -> None:
    """`--gpus N` with N > 1 outside torchrun: re-launch this command as N ranks
    (one process per GPU) through torch.distributed.run on 127.0.0.1.  Under
    torchrun the world size must equal --gpus: a mismatch fails loudly instead
    of timing another number of GPUs than the line claims."""
    world = os.environ.get("WORLD_SIZE")
    if world is not None:
        if int(world) != args.gpus:
            raise SystemExit(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}")
        return
    if args.gpus <= 1:
        return
    os.environ.setdefault("NCCL_DEBUG", "INFO")  # the communicator's rank count is in the log
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__),
           *sys.argv[1:]]
    print(f"bench.py: launching {args.gpus} ranks: {' '.join(cmd)}", file=sys.stderr, flush=True)
    os.execv(sys.executable, cmd)


def main():
    args = parse()
    launch_ranks(args)
    D = Dist()
    if args.impl == "reference":
        run_reference(args, D)
        return
    run_ours(args, D)
    if D.pg:
        D.pg.destroy_process_group()


if __name__ == "__main__":
    main()
