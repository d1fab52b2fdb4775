"""Row-range sharding and the tiny per-query exchanges.

The paper runs on one GPU (Table II); sharding is this build's
extension.  Each rank owns a contiguous row range; the only collectives are

* SELECT: all_gather of one int64 count per rank -> exclusive scan -> the
  rank's global output offset (outputs stay sharded at known positions).  For
  device tensors the scan is libra.so's ``ra_select_offsets`` kernel (stream
  ordered, no host round trip); for host tensors it is plain integer code;
* Q1: all_gather of the 400-byte ``ra_q1_partial`` of each rank (NCCL has no
  128-bit sum), merged exactly by ``ra_q1_finalize``.

torch.distributed is plumbing only (NCCL on the GPU box, gloo in CPU tests and
in the 2-rank tests that share one GPU).
"""
from __future__ import annotations


def shard_range(n: int, rank: int, world: int, align: int = 4) -> tuple[int, int]:
    """Rows [lo, hi) of ``rank``: contiguous, covering [0, n), boundaries rounded
    down to multiples of ``align`` rows (keeps 16-B alignment of int32 shards)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")

    def cut(r):
        if r >= world:
            return n
        c = (n * r // world) // align * align
        return min(c, n)

    return cut(rank), cut(rank + 1)


def exclusive_offsets(counts) -> list[int]:
    out, run = [], 0
    for c in counts:
        out.append(run)
        run += int(c)
    return out


def _all_gather(out, inp, group=None):
    """all_gather_into_tensor; gloo with device tensors is staged through host
    memory (gloo is the CPU-test / shared-GPU functional backend only)."""
    import torch.distributed as dist
    if inp.is_cuda and dist.get_backend(group) == "gloo":
        tmp = out.cpu()
        dist.all_gather_into_tensor(tmp, inp.cpu(), group=group)
        out.copy_(tmp)
    else:
        dist.all_gather_into_tensor(out, inp, group=group)
    return out


def exchange_counts(count, group=None, counts=None, offsets=None, total=None):
    """all_gather one int64 count per rank, then the exclusive scan.

    Returns ``(counts, offset, total)``: the gathered counts (int64[world]),
    this rank's global output offset and the global count.  Device tensors
    stay on the device (0-dim views, not synchronised); ``counts``,
    ``offsets`` (int64[world]) and ``total`` (int64[1]) may be preallocated."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    dev = count.device
    if counts is None:
        counts = torch.empty(world, dtype=torch.int64, device=dev)
    _all_gather(counts, count.reshape(1).to(torch.int64), group)
    if counts.is_cuda:
        from . import _ra
        if offsets is None:
            offsets = torch.empty(world, dtype=torch.int64, device=dev)
        if total is None:
            total = torch.empty(1, dtype=torch.int64, device=dev)
        _ra.ra_select_offsets(counts.data_ptr(), world, offsets.data_ptr(), total.data_ptr(),
                              int(torch.cuda.current_stream(dev).cuda_stream))
        return counts, offsets[rank], total[0]
    host = [int(c) for c in counts.tolist()]
    offs = exclusive_offsets(host)
    return counts, torch.tensor(offs[rank], dtype=torch.int64), torch.tensor(sum(host), dtype=torch.int64)


def gather_partials(partial, group=None):
    """all_gather each rank's ra_q1_partial bytes (uint8 tensor) — the Q1 exchange."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    out = torch.empty(world * partial.numel(), dtype=torch.uint8, device=partial.device)
    return _all_gather(out, partial, group)


def gather_outputs(out, count, offsets, total, root: int = 0, group=None):
    """Optional concatenation of the sharded SELECT output onto one rank
    (SURVEY §8(e)): rank r sends its rows out[:count_r] to `root`, which
    receives them at their global offsets (from ``exchange_counts``) into one
    tensor of ``total`` rows, in rank order — equal to the 1-GPU result.
    Point-to-point transfers (NCCL send/recv over NVLink on the GPU box, gloo
    in tests).  Returns the concatenation on `root`, None elsewhere."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    c = int(count)
    staged = out.is_cuda and dist.get_backend(group) == "gloo"  # gloo: point-to-point on host tensors
    if rank != root:
        if c:
            dist.send(out[:c].cpu() if staged else out[:c].contiguous(), dst=root, group=group)
        return None
    offs = [int(v) for v in (offsets.tolist() if hasattr(offsets, "tolist") else offsets)]
    tot = int(total)
    bounds = offs[1:] + [tot]
    full = torch.empty(max(1, tot), dtype=out.dtype, device=out.device)[:tot]
    full[offs[root]:offs[root] + c].copy_(out[:c])
    for r in range(world):
        if r != root and bounds[r] > offs[r]:
            if staged:
                tmp = torch.empty(bounds[r] - offs[r], dtype=out.dtype)
                dist.recv(tmp, src=r, group=group)
                full[offs[r]:bounds[r]].copy_(tmp)
            else:
                dist.recv(full[offs[r]:bounds[r]], src=r, group=group)
    return full
