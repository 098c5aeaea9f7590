"""GPU parity of word mode (gem_isa.h "WRD1", gem_words.cuh): the single-stream
path that runs each partition's AND list one signal per shared-memory word in
barrier-separated steps.  Bar as everywhere: bit-exact PO
and flop traces vs the CPU oracle; and word mode == the bit-packed boomerang
path (GEM_F_NO_WORDS) on the same blob, state and RAM contents included.
"""
import numpy as np
import pytest

from gen import stimulus
from gen.stimulus import stim_random
from oracle import Oracle
from tests import circuits
from tests.common import blob, eaig
from tests.test_gpu import _full_parity

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gem():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    from paper_conf_dac_guozwlr25_b200 import gem as g
    return g


@pytest.mark.parametrize("cfg", ["c1", "c2", "c3"])
def test_word_mode_is_the_single_stream_path(gem, cfg):
    sim = gem.Simulator(blob(cfg))
    assert sim.info["words"] == 1 and sim.info["lanes"] == 0
    bits = gem.Simulator(blob(cfg), flags=gem.GEM_F_NO_WORDS)
    assert bits.info["words"] == 0


@pytest.mark.parametrize("cfg,T", [("c1", 3000), ("c3", 400)])
def test_bit_packed_path_still_exact(gem, cfg, T):
    """The paper's boomerang-layer path (GEM_F_NO_WORDS) stays parity-green."""
    n_pi = Oracle(eaig(cfg)).n_pi
    _full_parity(gem, eaig(cfg), blob(cfg), stimulus(cfg, n_pi, T), extra_flags=gem.GEM_F_NO_WORDS)


def test_c3_word_mode_equals_bit_mode(gem):
    T = 500
    st = stimulus("c3", 256, T)
    w = gem.Simulator(blob("c3"))
    b = gem.Simulator(blob("c3"), flags=gem.GEM_F_NO_WORDS)
    assert w.info["words"] == 1 and b.info["words"] == 0
    assert np.array_equal(w.run(st), b.run(st))
    assert np.array_equal(w.read_state(), b.read_state())
    for ram in range(w.info["n_rams"]):
        assert np.array_equal(w.read_ram(ram), b.read_ram(ram))


@pytest.mark.parametrize("opts,kw", [("parts=1", {}), ("parts=5", {}), ("parts=5 stages=2", {}),
                                     ("parts=4 stages=2 cut_level=3", {}), ("parts=3 word_step=32", {}),
                                     ("parts=5", {"grid_limit": 2}), ("parts=5", {"grid_limit": 1}),
                                     ("parts=4", {"n_streams": 3})])
def test_word_mode_small_designs(gem, tmp_path, opts, kw):
    """RAM blocks, one and two stages, narrow steps (word_step=32), several work
    items per CTA (grid_limit 2, a single CTA running every partition with the
    flops in shared memory), and 3 streams."""
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.small_G(seed=21, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    S = kw.get("n_streams", 1)
    st = np.stack([stim_random(net.n_pi, 300, 3 + s, reset_pi0_cycles=2) for s in range(S)])
    b = compile_file(p, opts + " words=1")
    sim = _full_parity(gem, p, b, st if S > 1 else st[0], **kw)
    assert sim.info["words"] == 1


def test_word_mode_cells_ram_shift(gem, tmp_path):
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    rng = np.random.default_rng(11)
    for name, net in [("cells", circuits.cells()), ("ram", circuits.ram_direct()),
                      ("sr", circuits.shift_register(70)), ("rc", circuits.random_comb(12, 400, 30, 9)),
                      ("cnt", circuits.counter_with_load())]:
        p = circuits.save(net, str(tmp_path), name)
        n_pi = Oracle(p).n_pi
        st = rng.integers(0, 1 << 32, size=(300, (n_pi + 31) // 32), dtype=np.uint64).astype(np.uint32)
        if n_pi % 32:
            st[:, -1] &= (1 << (n_pi % 32)) - 1
        if name == "ram":
            st[:, 0] = (st[:, 0] & ~np.uint32(0x3FFFFFF)) | (st[:, 0] & 0x7) | ((st[:, 0] & 0x7) << 13)
        sim = _full_parity(gem, p, compile_file(p, "words=1"), st, chunks=(1, 37, 150))
        assert sim.info["words"] == 1, name


def test_word_mode_ram_preload_and_resume(gem, tmp_path):
    """RAM preloaded before the first cycle (U10) and a state written between
    steps: word mode reads both (Q / RD re-enter its shared-memory copy)."""
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.ram_direct()
    p = circuits.save(net, str(tmp_path), "ram")
    o = Oracle(p)
    rng = np.random.default_rng(3)
    T = 200
    st = rng.integers(0, 1 << 32, size=(T, (o.n_pi + 31) // 32), dtype=np.uint64).astype(np.uint32)
    if o.n_pi % 32:
        st[:, -1] &= (1 << (o.n_pi % 32)) - 1
    words = rng.integers(0, 1 << 32, size=8192, dtype=np.uint64).astype(np.uint32)
    for blob_opts in ("words=1", "parts=2 words=1"):
        sim = gem.Simulator(compile_file(p, blob_opts))
        assert sim.info["words"] == 1
        sim.write_ram(0, words)
        o2 = Oracle(p)
        o2.set_ram(0, words)
        r = o2.run(st, state=True)
        po = sim.run(st[:90])
        q = sim.read_state()
        sim.write_state(q)           # round trip between steps
        po2 = sim.run(st[90:])
        assert np.array_equal(np.concatenate([po[0], po2[0]]), r["po"]), blob_opts
        assert np.array_equal(sim.read_ram(0), o2.get_ram(0)), blob_opts


def test_c3_word_mode_2000_cycles_checkpoints(gem):
    """C3 in word mode: PO trace and per-cycle flop digest over 2,000 cycles in
    ragged launches, final flops and RAM contents (the bench's path)."""
    T = 2000
    st = stimulus("c3", 256, T)
    sim = gem.Simulator(blob("c3"), flags=gem.GEM_F_DIGEST)
    assert sim.info["words"] == 1
    po, dg = [], []
    for a, e in [(0, 1), (1, 700), (700, 1337), (1337, 2000)]:
        sim.set_inputs(st[a:e])
        sim.step(e - a)
        po.append(sim.read_outputs(e - a)[0])
        dg.append(sim.read_digests(e - a)[0])
    o = Oracle(eaig("c3"))
    r = o.run(st, digest=True)
    assert np.array_equal(np.concatenate(po), r["po"])
    assert np.array_equal(np.concatenate(dg), r["digest"])
    assert np.array_equal(sim.read_state()[0], o.get_state())
    for ram in range(o.n_rams):
        assert np.array_equal(sim.read_ram(ram), o.get_ram(ram))


def test_c2_two_stage_word_mode(gem):
    """C2 mapped as two stages (P:109 cut words exchanged through the second
    grid barrier) in word mode: PO and flops every cycle vs the oracle."""
    from tests.common import MAP_OPTS
    b = blob("c2", MAP_OPTS["c2"] + " stages=2")
    sim = _full_parity(gem, eaig("c2"), b, stimulus("c2", 128, 600), chunks=(250,))
    assert sim.info["words"] == 1 and sim.info["n_stages"] == 2


def test_c3_word_mode_four_streams(gem):
    """Four independent streams of C3 in word mode (several work items per
    CTA, the generic item loop): every stream's PO trace and final flops equal
    its own oracle run."""
    S, T = 4, 120
    st = np.stack([stimulus("c3", 256, T, seed=300 + s) for s in range(S)])
    sim = gem.Simulator(blob("c3"), n_streams=S)
    assert sim.info["words"] == 1
    po = sim.run(st)
    q = sim.read_state()
    for s in range(S):
        o = Oracle(eaig("c3"))
        r = o.run(st[s])
        assert np.array_equal(po[s], r["po"]), s
        assert np.array_equal(q[s], o.get_state()), s
