"""GPU parity of the multi-rank path through the CUDA
kernels: two ranks (gloo, both on cuda:0 — the GPU box has one GPU; NCCL needs
one per rank) each run ra_select_chain / ra_q1 on their own row range, exchange
counts (all_gather + libra.so's ra_select_offsets) and Q1 partials
(all_gather + ra_q1_finalize's exact merge).  Each rank's SELECT output placed
at its global offset, concatenated, must equal the oracle's SELECT over the
whole column element by element; the merged Q1 must equal the oracle's Q1."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import oracle
import ragen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ("count_order", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "sum_disc",
        "avg_qty", "avg_price", "avg_disc")


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, n, m, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_wudwcyc12_b200 as R
        from paper_conf_ipps_wudwcyc12_b200 import dist as rdist
        torch.cuda.set_device(0)
        sh = int(torch.cuda.current_stream().cuda_stream)
        # ---- SELECT chain on this rank's rows of one seeded column
        lo, hi = rdist.shard_range(n, rank, world)
        x = torch.empty(hi - lo, dtype=torch.int32, device="cuda")
        ragen.int32_column_dev(61, x, row0=lo, stream=sh)
        preds = [("lt", t) for t in ragen.nested_thresholds(0.5, 2)] + [("ne", 12345)]
        out, cnt = R.select_chain(x, preds)
        counts, off, total = rdist.exchange_counts(cnt)
        c, o, t = int(cnt.item()), int(off.item()), int(total.item())
        placed = torch.zeros(t, dtype=torch.int32)
        placed[o:o + c] = out[:c].cpu()
        dist.all_reduce(placed)  # assemble the sharded output (checking only)
        whole = oracle.select(ragen.int32_column(61, n), preds)
        ok_select = placed.numel() == whole.size and bool(np.array_equal(placed.numpy(), whole))
        host_offs = rdist.exclusive_offsets(counts.tolist())
        ok_offsets = o == host_offs[rank] and t == sum(counts.tolist())
        offs_dev = torch.tensor(host_offs, dtype=torch.int64, device="cuda")
        full = rdist.gather_outputs(out, c, offs_dev, t)  # concatenation onto rank 0
        ok_select &= (full is None) if rank != 0 else bool(np.array_equal(full.cpu().numpy(), whole))
        # ---- Q1 on this rank's rows of one lineitem table
        a, b = rdist.shard_range(m, rank, world)
        cols = ragen.lineitem(62, m, 20000)
        dcols = {k: torch.from_numpy(np.ascontiguousarray(v[a:b])).cuda() for k, v in cols.items()}
        part = R.q1(dcols)
        gathered = rdist.gather_partials(part)
        merged, rc = R.q1_finalize(bytes(gathered.cpu().numpy().tobytes()))
        exp, _ = oracle.q1(cols, R.Q1_CUTOFF_DELTA90)
        ok_q1 = rc == R.RA_OK and len(merged) == len(exp) and all(
            g[k] == e[k] for g, e in zip(merged, exp) for k in KEYS)
        q.put((rank, ok_select, ok_offsets, ok_q1, c, o, t))
    except Exception as e:  # report, do not hang the parent
        q.put((rank, False, False, False, repr(e), 0, 0))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n,m", [(100_003, 50_001), ((1 << 24) + 5, 3_000_007)])
def test_two_ranks_through_the_kernels(n, m):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n, m, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=600) for _ in range(2))
    for p in procs:
        p.join(timeout=120)
    assert all(r[1] and r[2] and r[3] for r in res), res
    assert res[0][5] == 0 and res[1][5] == res[0][4]  # rank 1 starts where rank 0 ends


@pytest.mark.parametrize("world", [1, 2, 3, 31, 32, 33, 100, 1000, 65536])
def test_select_offsets_kernel(world):
    import paper_conf_ipps_wudwcyc12_b200 as R
    g = torch.Generator().manual_seed(world)
    counts = torch.randint(0, 1 << 40, (world,), generator=g, dtype=torch.int64)
    d = counts.cuda()
    offs = torch.full((world,), -1, dtype=torch.int64, device="cuda")
    tot = torch.full((1,), -1, dtype=torch.int64, device="cuda")
    R.ra_select_offsets(d.data_ptr(), world, offs.data_ptr(), tot.data_ptr(),
                        int(torch.cuda.current_stream().cuda_stream))
    run, exp = 0, []
    for c in counts.tolist():
        exp.append(run)
        run += c
    assert offs.cpu().tolist() == exp and int(tot.item()) == run


def test_select_offsets_rejects_bad_sizes():
    import paper_conf_ipps_wudwcyc12_b200 as R
    d = torch.zeros(4, dtype=torch.int64, device="cuda")
    for bad in (0, -1, R.RA_MAX_RANKS + 1):
        with pytest.raises(R.RAError) as e:
            R.ra_select_offsets(d.data_ptr(), bad, d.data_ptr(), 0, 0)
        assert e.value.code == R.RA_E_INVAL


def test_bench_launches_ranks_itself():
    """`bench.py --gpus 2` without torchrun re-launches itself as two ranks
    (gloo here: the box has one GPU) and reports n_gpus == 2."""
    env = dict(os.environ, RA_BENCH_BACKEND="gloo")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "5",
                        "--warmup", "3", "--no-extras", "--rows-log2", "24"],
                       capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["value"] > 0 and line["gpu_launches"] >= 5
