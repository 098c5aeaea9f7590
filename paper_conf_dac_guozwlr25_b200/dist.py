"""Multi-GPU plumbing.

Batched stimuli: independent stimulus streams over the same
design shard naturally: rank g simulates streams [start_g, start_g + count_g)
with no per-cycle communication, and after a step the PO traces are gathered
to rank 0 over NCCL (NVLink/NVSwitch).

Single design split over devices (PAPER.md P:247 lists
multi-GPU as future work): every rank loads the same blob with dist_world /
dist_rank, the kernels exchange the committed words over peer memory and meet
at a cross-device barrier each stage (include/gem.h gem_dist_*).  This module
only wires the handles: connect_split exchanges CUDA IPC handles of the ranks'
buffers over torch.distributed (one process per GPU), connect_local connects
handles of one process (several devices, or one device in tests).

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


# ---- single design split over devices (gem_dist_*) -------------------------
def connect_split(sim, max_cycles: int, group: Optional[dist.ProcessGroup] = None):
    """One process per rank: export this rank's buffers, all-gather their CUDA
    IPC handles, map every peer's and connect.  Collective over `group`; the
    rank order of `group` must match the handles' dist_rank."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    sim.dist_export(max_cycles)
    mine = sim.dist_ipc_handles()
    handles: List[Optional[bytes]] = [None] * world
    dist.all_gather_object(handles, mine, group=group)
    peers = [None if r == rank else sim.dist_ipc_open(handles[r]) for r in range(world)]
    sim.dist_connect(peers)
    dist.barrier(group=group)   # nobody steps before every rank is connected
    return peers


def connect_local(sims, max_cycles: int):
    """Handles of one process (sims[r] = rank r): export all, connect each."""
    bufs = [s.dist_export(max_cycles) for s in sims]
    for s in sims:
        s.dist_connect(bufs)
    return bufs


def step_local(sims, ncycles: int):
    """Step the ranks of one process together (their kernels meet at the
    cross-device barrier, so each launch must be asynchronous: GEM_F_ASYNC)."""
    from .gem import GEM_F_ASYNC
    for s in sims:
        if not s.flags & GEM_F_ASYNC:
            raise ValueError("in-process ranks need GEM_F_ASYNC (the launches must overlap)")
    for s in sims:
        s.step(ncycles)
    return [s.last_step_ms() for s in sims]
