"""Multi-GPU batched-stimulus plumbing.

Single designs are replicas only (per-cycle partition exchange stays on one
GPU, PAPER.md P:247 lists multi-GPU as future work).  Independent stimulus
streams over the same design shard naturally: rank g simulates streams
[start_g, start_g + count_g) with no per-cycle communication, and after a
step the PO traces are gathered to rank 0 over NCCL (NVLink/NVSwitch).

torch.distributed is plumbing only; the simulation runs in libgem.
"""
from __future__ import annotations

from typing import List, Optional, Tuple

import torch
import torch.distributed as dist


def shard_streams(total: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous, balanced shard of `total` global stream ids for `rank`."""
    if world < 1 or not (0 <= rank < world) or total < 0:
        raise ValueError("bad shard request")
    base, extra = divmod(total, world)
    count = base + (1 if rank < extra else 0)
    start = rank * base + min(rank, extra)
    return start, count


def gather_traces(local: torch.Tensor, total_streams: int, dst: int = 0,
                  group: Optional[dist.ProcessGroup] = None) -> Optional[torch.Tensor]:
    """Gather per-rank traces [count_g, ...] into [total_streams, ...] on `dst`.

    Shards may be uneven; each rank pads to the largest shard so a single
    collective (gather) moves everything.  Returns the full tensor on `dst`,
    None elsewhere.  Works with NCCL (CUDA tensors) and gloo (CPU tensors).
    """
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    counts = [shard_streams(total_streams, world, r)[1] for r in range(world)]
    mx = max(counts)
    if local.shape[0] != counts[rank]:
        raise ValueError(f"rank {rank}: local trace has {local.shape[0]} streams, expected {counts[rank]}")
    pad = local
    if local.shape[0] < mx:
        pad = torch.zeros((mx,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
        pad[:local.shape[0]] = local
    bufs: Optional[List[torch.Tensor]] = None
    if rank == dst:
        bufs = [torch.empty_like(pad) for _ in range(world)]
    dist.gather(pad, bufs, dst=dst, group=group)
    if rank != dst:
        return None
    return torch.cat([b[:c] for b, c in zip(bufs, counts)], 0)
