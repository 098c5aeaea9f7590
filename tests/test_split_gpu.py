"""Row f4: one design split over devices (include/gem.h gem_dist_*), parity vs the oracle.

The test box has one GPU, so the ranks are several handles on cuda:0: in one
process (dist.connect_local: raw device pointers, asynchronous launches that
meet at the cross-device barrier) and in two processes (dist.connect_split:
CUDA IPC handles exchanged over gloo).  The kernel path is the one a
multi-GPU run takes (peer stores of every committed Q / RD / cut / PO word,
system-scope flag barrier); only the peer memory is local.  Every rank's PO
trace and flop trace must equal the oracle's (PAPER.md P:194-196 commit
semantics: the trace is unique).
"""
import os
import socket

import numpy as np
import pytest

from gen import stimulus
from gen.stimulus import stim_random
from oracle import Oracle
from tests import circuits
from tests.common import blob, eaig

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gem():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    from paper_conf_dac_guozwlr25_b200 import gem as g
    return g


def _split_parity(gem, path, b, stim, world, chunks=(None,), n_streams=1, grid_limit=8):
    from paper_conf_dac_guozwlr25_b200.dist import connect_local, step_local
    T = stim.shape[-2]
    flags = gem.GEM_F_TRACE_STATE | gem.GEM_F_DIGEST | gem.GEM_F_ASYNC
    sims = [gem.Simulator(b, n_streams=n_streams, flags=flags, grid_limit=grid_limit, dist_world=world, dist_rank=r)
            for r in range(world)]
    bounds = [0, T] if chunks == (None,) else [0, *chunks, T]
    connect_local(sims, max(e - a for a, e in zip(bounds[:-1], bounds[1:])))
    po = [[] for _ in sims]
    st = [[] for _ in sims]
    for a, e in zip(bounds[:-1], bounds[1:]):
        for s in sims:
            s.set_inputs(stim[..., a:e, :])
        step_local(sims, e - a)
        for r, s in enumerate(sims):
            po[r].append(s.read_outputs(e - a))
            st[r].append(s.read_state_trace(e - a))
    stims = stim if stim.ndim == 3 else stim[None]
    refs = [Oracle(path).run(stims[k], state=True) for k in range(n_streams)]
    for r in range(world):
        p, q = np.concatenate(po[r], 1), np.concatenate(st[r], 1)
        for k in range(n_streams):
            assert np.array_equal(p[k], refs[k]["po"]), ("PO", r, k, np.where((p[k] != refs[k]["po"]).any(1))[0][:5])
            assert np.array_equal(q[k], refs[k]["state"]), ("Q", r, k)
    return sims


def test_split_small_ram_designs(gem, tmp_path):
    """RAM blocks (RD words cross ranks), one and two stages (cut words cross
    ranks inside a cycle), 2 and 3 ranks, ragged steps, 3 streams."""
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.small_G(seed=21, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    st = stim_random(net.n_pi, 300, 3, reset_pi0_cycles=2)
    for opts, world in [("parts=5", 2), ("parts=5", 3), ("parts=5 stages=2", 2), ("parts=8 stages=2", 4)]:
        b = compile_file(p, opts)
        own = gem.dist_owner(b, world)
        assert len(set(own.tolist())) == world          # every rank has work
        _split_parity(gem, p, b, st, world, chunks=(1, 40, 41))
    st3 = np.stack([stim_random(net.n_pi, 120, s, reset_pi0_cycles=2) for s in (4, 5, 6)])
    _split_parity(gem, p, compile_file(p, "parts=5 stages=2"), st3, 2, n_streams=3)


def test_split_c2_and_one_partition(gem):
    """C2 (about 50 partitions) over 2 ranks for 2000 cycles; C1 (one
    partition) over 2 ranks: rank 1 owns nothing and still meets every barrier."""
    _split_parity(gem, eaig("c2"), blob("c2"), stimulus("c2", 128, 2000), 2, chunks=(700,), grid_limit=16)
    _split_parity(gem, eaig("c1"), blob("c1"), stimulus("c1", 35, 500), 2)


def test_split_guards(gem):
    """A dist handle refuses gem_step before gem_dist_connect and more cycles per
    step than gem_dist_export's max_cycles; a plain handle cannot export."""
    from paper_conf_dac_guozwlr25_b200.dist import connect_local
    b = blob("c1")
    s0 = gem.Simulator(b, flags=gem.GEM_F_ASYNC, dist_world=2, dist_rank=0)
    s1 = gem.Simulator(b, flags=gem.GEM_F_ASYNC, dist_world=2, dist_rank=1)
    s0.set_inputs(stimulus("c1", 35, 20))
    with pytest.raises(gem.GemError, match="INVAL"):
        s0.step(5)
    connect_local([s0, s1], 10)
    with pytest.raises(gem.GemError, match="max_cycles"):
        s0.step(20)
    with pytest.raises(gem.GemError, match="not a dist handle"):
        gem.Simulator(b).dist_export(10)
    with pytest.raises(gem.GemError, match="INVAL"):
        gem.Simulator(b, dist_world=2, dist_rank=2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


T_IPC = 60


def _ipc_worker(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_dac_guozwlr25_b200 import gem
    from paper_conf_dac_guozwlr25_b200.dist import connect_split
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        sim = gem.Simulator(blob("c2"), flags=gem.GEM_F_TRACE_STATE, grid_limit=4, dist_world=world,
                            dist_rank=rank)
        connect_split(sim, T_IPC)
        sim.set_inputs(stimulus("c2", 128, T_IPC))
        sim.step(T_IPC)
        q.put((rank, sim.read_outputs(T_IPC), sim.read_state_trace(T_IPC)))
        dist.barrier()   # keep the mapped peer buffers alive until both have read
        sim.close()
    finally:
        dist.destroy_process_group()


def test_split_two_processes_ipc(gem):
    """Two processes (one per rank, as on a multi-GPU box) connected by CUDA IPC
    handles exchanged over torch.distributed: both traces equal the oracle's."""
    import torch.multiprocessing as mp
    blob("c2")   # map once, before the workers start
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = {}
    for _ in range(2):
        r, po, stt = q.get(timeout=600)
        res[r] = (po, stt)
    for pr in procs:
        pr.join(timeout=120)
        assert pr.exitcode == 0
    ref = Oracle(eaig("c2")).run(stimulus("c2", 128, T_IPC), state=True)
    for r in range(2):
        assert np.array_equal(res[r][0][0], ref["po"]), r
        assert np.array_equal(res[r][1][0], ref["state"]), r
