"""Multi-process (world size 2 and 3, gloo on CPU) checks of the batched-stream
sharding and trace gather used by bench.py for N>1 GPUs:
the gathered traces are identical for every world size."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_dac_guozwlr25_b200.dist import gather_traces, shard_streams


def test_shard_streams_cover_exactly():
    for total in (0, 1, 7, 64, 4096, 4097):
        for world in (1, 2, 3, 4, 8):
            seen = []
            for r in range(world):
                s, c = shard_streams(total, world, r)
                seen.extend(range(s, s + c))
            assert seen == list(range(total))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _trace_of(stream_ids, T, W):
    """Deterministic per-stream fake PO trace (stands in for libgem output)."""
    out = np.zeros((len(stream_ids), T, W), np.int32)
    for k, s in enumerate(stream_ids):
        rng = np.random.default_rng(1000 + s)
        out[k] = rng.integers(-2**31, 2**31 - 1, size=(T, W), dtype=np.int64).astype(np.int32)
    return out


def _worker(rank, world, port, total, T, W, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        s, c = shard_streams(total, world, rank)
        local = torch.from_numpy(_trace_of(range(s, s + c), T, W))
        full = gather_traces(local, total)
        if rank == 0:
            q.put(full.numpy())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,total", [(2, 64), (3, 37)])
def test_gather_traces_world_sizes(world, total):
    T, W = 5, 8
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, total, T, W, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert np.array_equal(got, _trace_of(range(total), T, W))


# ---- row f4: handle exchange of a design split over ranks (host logic) -----
class _FakeSplitSim:
    """Stands in for gem.Simulator's gem_dist_* calls (no GPU here)."""

    def __init__(self, rank):
        self.rank, self.calls, self.connected = rank, [], None

    def dist_export(self, max_cycles):
        self.calls.append(("export", max_cycles))

    def dist_ipc_handles(self):
        return bytes([self.rank + 1]) * 328

    def dist_ipc_open(self, h):
        assert len(h) == 328 and len(set(h)) == 1
        self.calls.append(("open", h[0] - 1))
        return ("mapped", h[0] - 1)

    def dist_connect(self, peers):
        self.connected = list(peers)


def _split_worker(rank, world, port, q):
    from paper_conf_dac_guozwlr25_b200.dist import connect_split
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        s = _FakeSplitSim(rank)
        connect_split(s, 77)
        q.put((rank, s.calls, s.connected))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_connect_split_exchanges_every_peer(world):
    """dist.connect_split: each rank exports once, maps every OTHER rank's IPC
    handles (its own never) and connects with peers in rank order."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_split_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict((r, (c, con)) for r, c, con in (q.get(timeout=120) for _ in range(world)))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for r in range(world):
        calls, con = got[r]
        assert calls[0] == ("export", 77)
        assert sorted(c[1] for c in calls[1:]) == [x for x in range(world) if x != r]
        assert con == [None if x == r else ("mapped", x) for x in range(world)]


def test_dist_owner_split():
    """gem_dist_owner (host-only): every partition gets one rank < world, the
    split is deterministic, world 1 is all rank 0, and per stage the loads
    differ by at most one partition's cost (LPT)."""
    from paper_conf_dac_guozwlr25_b200 import gem, isa
    from tests.common import blob
    b = blob("c2")
    info = isa.blob_info(b)
    stages = [[p for p in range(info.n_parts) if info.part_stage[p] == s] for s in range(info.n_stages)]
    for world in (1, 2, 3, 8):
        own = gem.dist_owner(b, world)
        assert len(own) == info.n_parts and own.max() < world
        assert np.array_equal(own, gem.dist_owner(b, world))
        if world == 1:
            assert not own.any()
        for st in stages:
            cost = {p: max(int(info.part_cost[p]), 1) for p in st}
            load = [sum(cost[p] for p in st if own[p] == r) for r in range(world)]
            assert max(load) - min(load) <= max(cost.values())
    with pytest.raises(gem.GemError):
        gem.dist_owner(b[:-4], 2)
