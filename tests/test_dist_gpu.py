"""Batched streams sharded over ranks with REAL libgem output:
G gloo ranks (processes) share the one GPU of the test box, each simulates its
contiguous shard of the C5 streams through the C ABI, and the PO traces and
final flop states gathered to rank 0 are byte-identical to one process
simulating all streams (G = 2, 4, 8).  The bench's NCCL path uses the same
shard_streams / gather_traces code with CUDA tensors."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

TOTAL, T = 512, 40


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _inputs(streams):
    from gen import stimulus_streams
    return stimulus_streams("c5", 256, T, streams)


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    from paper_conf_dac_guozwlr25_b200 import gem
    from paper_conf_dac_guozwlr25_b200.dist import gather_traces, shard_streams
    from tests.common import blob
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        s0, n = shard_streams(TOTAL, world, rank)
        sim = gem.Simulator(blob("c5"), device=0, n_streams=n)
        po = sim.run(_inputs(range(s0, s0 + n)))
        q_state = sim.read_state()
        lanes = sim.info["lanes"]
        full_po = gather_traces(torch.from_numpy(po.view(np.int32)), TOTAL)
        full_q = gather_traces(torch.from_numpy(q_state.view(np.int32)), TOTAL)
        if rank == 0:
            q.put((full_po.numpy().view(np.uint32), full_q.numpy().view(np.uint32), lanes))
    finally:
        dist.destroy_process_group()


@pytest.fixture(scope="module")
def single():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    from paper_conf_dac_guozwlr25_b200 import gem
    from tests.common import blob
    sim = gem.Simulator(blob("c5"), device=0, n_streams=TOTAL)
    po = sim.run(_inputs(range(TOTAL)))
    return po, sim.read_state()


@pytest.mark.parametrize("world", [2, 4, 8])
def test_sharded_streams_gather_equals_single_process(single, world):
    import torch.multiprocessing as mp
    from tests.common import blob
    blob("c5")                         # map once (cached on disk) before the ranks start
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    po, qs, lanes = q.get(timeout=600)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    assert lanes == 1                  # every shard (>= 64 streams) runs in lane mode
    assert np.array_equal(po, single[0])
    assert np.array_equal(qs, single[1])
