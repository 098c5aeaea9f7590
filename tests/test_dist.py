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
