"""World-size-2 gloo tests (CPU) of the multi-GPU host logic: row-range shard
bounds, the SELECT count exchange -> global offsets, and the exact Q1 partial
merge.  The per-shard compute here is the oracle (the GPU kernels need a B200);
what is under test is the product's sharding/exchange/merge code."""
import ctypes
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import ragen

R = pytest.importorskip("paper_conf_ipps_wudwcyc12_b200")
from paper_conf_ipps_wudwcyc12_b200 import dist as rdist  # noqa: E402

SLOT = {(ord(rf), ord(ls)): 2 * i + j for i, rf in enumerate("ANR") for j, ls in enumerate("FO")}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_shard_range_covers_and_aligns():
    for n in (0, 1, 7, 1000, 1 << 20, 600_000_001):
        for world in (1, 2, 3, 8):
            parts = [rdist.shard_range(n, r, world) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            for (a, b), (c, d) in zip(parts[:-1], parts[1:]):
                assert b == c and a <= b
            for a, _ in parts:
                assert a % 4 == 0 or a == n
    assert rdist.exclusive_offsets([3, 0, 5, 2]) == [0, 3, 3, 8]


def _partial_from_rows(rows):
    p = R.ra_q1_partial()
    p.n_groups = 6
    for r in rows:
        g = p.group[SLOT[(r["rf_byte"], r["ls_byte"])]]
        g.count, g.sum_qty, g.sum_base_price, g.sum_disc = (
            r["count_order"], r["sum_qty"], r["sum_base_price"], r["sum_disc"])
        g.sum_disc_price_lo, g.sum_disc_price_hi = r["sum_disc_price"] & (2**64 - 1), r["sum_disc_price"] >> 64
        g.sum_charge_lo, g.sum_charge_hi = r["sum_charge"] & (2**64 - 1), r["sum_charge"] >> 64
    return bytes(p)


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # SELECT: shard, select, exchange counts, place at global offsets
        n = 100_003
        x = ragen.int32_column(21, n)
        preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)]
        lo, hi = rdist.shard_range(n, rank, world)
        mine = oracle.select(x[lo:hi], preds)
        counts, off, total = rdist.exchange_counts(torch.tensor([mine.size], dtype=torch.int64))
        placed = np.zeros(int(total), dtype=np.int32)
        placed[int(off):int(off) + mine.size] = mine
        buf = torch.from_numpy(placed)
        dist.all_reduce(buf)  # assemble for checking only
        whole = oracle.select(x, preds)
        ok_select = bool(np.array_equal(buf.numpy(), whole))
        # optional concatenation onto rank 0 (point-to-point), in rank order
        offs = rdist.exclusive_offsets(counts.tolist())
        full = rdist.gather_outputs(torch.from_numpy(np.ascontiguousarray(mine)), mine.size, offs, total)
        ok_select &= (full is None) if rank != 0 else bool(np.array_equal(full.numpy(), whole))
        # Q1: shard partials -> all_gather -> exact merge in ra_q1_finalize
        m = 200_001
        cols = ragen.lineitem(22, m, 20000)
        a, b = rdist.shard_range(m, rank, world)
        rows, _ = oracle.q1({k: v[a:b] for k, v in cols.items()}, 10471)
        part = torch.frombuffer(bytearray(_partial_from_rows(rows)), dtype=torch.uint8)
        gathered = rdist.gather_partials(part)
        merged, rc = R.q1_finalize(bytes(gathered.numpy().tobytes()))
        exp, _ = oracle.q1(cols, 10471)
        keys = ("count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc",
                "avg_qty", "avg_price", "avg_disc")
        ok_q1 = rc == R.RA_OK and len(merged) == len(exp) and all(
            g[k] == e[k] for g, e in zip(merged, exp) for k in keys)
        q.put((rank, ok_select, ok_q1, int(off), [int(c) for c in counts]))
    finally:
        dist.destroy_process_group()


def test_two_rank_exchange_and_merge():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert all(r[1] for r in res), res
    assert all(r[2] for r in res), res
    counts = res[0][4]
    assert [r[3] for r in res] == [0, counts[0]]


def test_bench_refuses_world_size_mismatch():
    """Under torchrun the world size must equal --gpus (else bench.py would time
    a different number of GPUs than its line claims)."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "1"], capture_output=True,
                       text=True, timeout=120, env=env)
    assert r.returncode != 0 and "WORLD_SIZE=2 but --gpus 1" in r.stderr


def test_exchange_counts_host_scan():
    """exchange_counts on host tensors uses plain integer code for the scan."""
    assert rdist.exclusive_offsets([]) == []
    assert rdist.exclusive_offsets([2**40, 1, 0]) == [0, 2**40, 2**40 + 1]


def test_bench_reference_arm_under_torchrun_two_ranks():
    """`bench.py --impl reference` launched the driver's way for N=2 (torchrun,
    127.0.0.1): rank 0 alone times the oracle and prints one JSON line with
    impl=reference, the other rank exits 0 without work.  CPU only."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(29500 + os.getpid() % 2000),
           os.path.join(root, "bench.py"), "--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "1",
           "--rows-log2", "18"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=300, cwd=root)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["unit"] == "rows/s" and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"
