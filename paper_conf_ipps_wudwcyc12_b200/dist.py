"""Row-range sharding and the tiny per-query exchanges.

The paper runs on one GPU (Table II); sharding is this build's
extension.  Each rank owns a contiguous row range; the only collectives are

* SELECT: all_gather of one int64 count per rank -> exclusive scan -> the
  rank's global output offset (outputs stay sharded at known positions);
* Q1: all_gather of the 400-byte ``ra_q1_partial`` of each rank (NCCL has no
  128-bit sum), merged exactly by ``ra_q1_finalize``.

torch.distributed is plumbing only (NCCL on the GPU box, gloo in CPU tests).
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


def exchange_counts(count, group=None, counts=None):
    """all_gather one int64 count per rank; returns (counts tensor, this rank's
    global offset, total) — the SELECT exchange (a9).  ``counts`` (int64[world],
    optional) receives the gathered counts."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    if counts is None:
        counts = torch.empty(world, dtype=torch.int64, device=count.device)
    dist.all_gather_into_tensor(counts, count.reshape(1).to(torch.int64), group=group)
    offs = torch.cumsum(counts, 0) - counts
    rank = dist.get_rank(group)
    return counts, offs[rank], counts.sum()


def gather_partials(partial, group=None):
    """all_gather each rank's ra_q1_partial bytes (uint8 tensor) — the Q1 exchange."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    out = torch.empty(world * partial.numel(), dtype=torch.uint8, device=partial.device)
    dist.all_gather_into_tensor(out, partial, group=group)
    return out
