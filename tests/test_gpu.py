"""GPU parity: the sm_100a path (through the C ABI) vs the CPU oracle, bit-exact.

Bar: the trace of an acyclic 2-state single-clock netlist is
unique, so every PO and flop must match the oracle at every cycle.
  C1, C2, small designs: full PO and full flop vector every cycle.
  C3, C5: full PO trace, per-cycle flop digest, final flops and RAM contents.
  C4: sampled (a short window; the oracle needs seconds per cycle there).
"""
import numpy as np
import pytest

from gen import stimulus, stimulus_streams
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


def _full_parity(gem, path, b, stim, n_streams=1, chunks=(None,), **kw):
    """Run GPU and oracle; compare PO + state trace every cycle."""
    T = stim.shape[-2]
    flags = gem.GEM_F_TRACE_STATE | gem.GEM_F_DIGEST | kw.pop("extra_flags", 0)
    sim = gem.Simulator(b, n_streams=n_streams, flags=flags, **kw)
    po_g, st_g, dg_g = [], [], []
    bounds = [0, T] if chunks == (None,) else [0, *chunks, T]
    for a, e in zip(bounds[:-1], bounds[1:]):
        sim.set_inputs(stim[..., a:e, :])
        sim.step(e - a)
        po_g.append(sim.read_outputs(e - a))
        st_g.append(sim.read_state_trace(e - a))
        dg_g.append(sim.read_digests(e - a))
    po_g = np.concatenate(po_g, 1)
    st_g = np.concatenate(st_g, 1)
    dg_g = np.concatenate(dg_g, 1)
    stims = stim if stim.ndim == 3 else stim[None]
    for s in range(n_streams):
        r = Oracle(path).run(stims[s], state=True, digest=True)
        assert np.array_equal(po_g[s], r["po"]), ("PO", s, np.where((po_g[s] != r["po"]).any(1))[0][:5])
        assert np.array_equal(st_g[s], r["state"]), ("Q", s, np.where((st_g[s] != r["state"]).any(1))[0][:5])
        assert np.array_equal(dg_g[s], r["digest"]), ("digest", s)
    return sim


def test_c1_full_10k_cycles(gem):
    _full_parity(gem, eaig("c1"), blob("c1"), stimulus("c1", 35, 10_000))


def test_c1_ragged_steps_and_resume(gem):
    # run(n)+run(m)+... == run(n+m+...) with ragged chunk sizes
    _full_parity(gem, eaig("c1"), blob("c1"), stimulus("c1", 35, 1000), chunks=(1, 2, 37, 500))


def test_small_designs_with_ram_and_stages(gem, tmp_path):
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.small_G(seed=21, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    st = stim_random(net.n_pi, 400, 3, reset_pi0_cycles=2)
    for opts in ["parts=1", "parts=5", "parts=5 stages=2", "parts=3 max_state_words=256"]:
        _full_parity(gem, p, compile_file(p, opts), st)


def test_cells_ram_shift(gem, tmp_path):
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    rng = np.random.default_rng(5)
    for name, net in [("cells", circuits.cells()), ("ram", circuits.ram_direct()),
                      ("sr", circuits.shift_register(70)), ("rc", circuits.random_comb(12, 400, 30, 9))]:
        p = circuits.save(net, str(tmp_path), name)
        n_pi = Oracle(p).n_pi
        st = rng.integers(0, 1 << 32, size=(300, (n_pi + 31) // 32), dtype=np.uint64).astype(np.uint32)
        if n_pi % 32:
            st[:, -1] &= (1 << (n_pi % 32)) - 1
        if name == "ram":
            st[:, 0] = (st[:, 0] & ~np.uint32(0x3FFFFFF)) | (st[:, 0] & 0x7) | ((st[:, 0] & 0x7) << 13)
        _full_parity(gem, p, compile_file(p), st)


def test_activity_pruning_gated_modules(gem, tmp_path):
    """Row f3 (GEM_F_ACTIVITY): partitions whose input ports did not
    change are skipped; every PO and flop stays bit-exact, and the idle
    modules' partition-cycles are actually skipped."""
    from gen.stimulus import stim_bursts
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.gated_counters(8, 16)
    p = circuits.save(net, str(tmp_path), "gated")
    T = 1000
    st = stim_bursts(8, T, 11)
    sim = _full_parity(gem, p, compile_file(p, "parts=8"), st, chunks=(1, 300), extra_flags=gem.GEM_F_ACTIVITY)
    ev, sk = sim.read_activity()
    n_parts = sim.info["n_parts"]
    assert n_parts >= 4 and sim.info["grid"] == n_parts
    assert ev + sk == n_parts * T          # every CTA runs one partition: all eligible
    assert sk > 0.5 * (ev + sk), (ev, sk)  # enables are on 8/64 of the cycles
    # the same design with inputs that change every cycle: nothing to skip
    rng = np.random.default_rng(3)
    st2 = rng.integers(0, 256, size=(200, 1)).astype(np.uint32)
    sim2 = _full_parity(gem, p, compile_file(p, "parts=8"), st2, extra_flags=gem.GEM_F_ACTIVITY)
    ev2, sk2 = sim2.read_activity()
    assert ev2 + sk2 == n_parts * 200 and sk2 < ev2


def test_activity_pruning_ram_stages_streamed(gem, tmp_path):
    """GEM_F_ACTIVITY on designs with RAM blocks, two stages, streamed programs
    (no residency) and multi-item CTAs: results equal the oracle's."""
    from gen.stimulus import hold
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.small_G(seed=21, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    st = hold(stim_random(net.n_pi, 100, 3, reset_pi0_cycles=2), 4)
    for opts, kw in [("parts=5", {}), ("parts=5 stages=2", {}), ("parts=5", {"grid_limit": 2})]:
        _full_parity(gem, p, compile_file(p, opts), st, chunks=(7, 200), extra_flags=gem.GEM_F_ACTIVITY, **kw)
    _full_parity(gem, p, compile_file(p, "parts=5"), st, extra_flags=gem.GEM_F_ACTIVITY | gem.GEM_F_NO_RESIDENT)
    _full_parity(gem, eaig("c1"), blob("c1"), hold(stimulus("c1", 35, 500), 3), extra_flags=gem.GEM_F_ACTIVITY)


def test_c2_full_parity(gem):
    """C2 (100K ANDs, 4K flops): full PO and flop vectors every cycle for 10,000
    cycles, in ragged gem_step chunks (SURVEY §8(c) protocol for C1-C2)."""
    _full_parity(gem, eaig("c2"), blob("c2"), stimulus("c2", 128, 10_000), chunks=(3000, 3001, 7777))


def test_c3_parity_digests_and_ram(gem):
    T = 600
    st = stimulus("c3", 256, T)
    sim = gem.Simulator(blob("c3"), flags=gem.GEM_F_DIGEST)
    sim.set_inputs(st)
    sim.step(T)
    po = sim.read_outputs(T)[0]
    dg = sim.read_digests(T)[0]
    o = Oracle(eaig("c3"))
    r = o.run(st, digest=True)
    assert np.array_equal(po, r["po"])
    assert np.array_equal(dg, r["digest"])
    assert np.array_equal(sim.read_state()[0], o.get_state())
    for ram in range(o.n_rams):
        assert np.array_equal(sim.read_ram(ram), o.get_ram(ram))


def test_c3_state_roundtrip_and_determinism(gem):
    T = 200
    st = stimulus("c3", 256, T)
    a = gem.Simulator(blob("c3"))
    b = gem.Simulator(blob("c3"))
    pa = a.run(st)
    pb = b.run(st)
    assert np.array_equal(pa, pb)
    q = a.read_state()
    c = gem.Simulator(blob("c3"))
    c.write_state(q)
    assert np.array_equal(c.read_state(), q)


def test_c3_speed_independent_of_stimulus(gem):
    """the method is oblivious -- every live AND is
    evaluated every cycle -- so cycles/s must not depend on the stimulus: two
    stimulus seeds (and an all-zero stimulus) time within 3% (median of 5)."""
    T = 1000
    sim = gem.Simulator(blob("c3"))
    times = {}
    for name, st in [("seed103", stimulus("c3", 256, T)), ("seed7", stimulus("c3", 256, T, seed=7)),
                     ("zeros", np.zeros((T, 8), np.uint32))]:
        ms = []
        for _ in range(5):
            sim.set_inputs(st)
            sim.step(T)
            ms.append(sim.last_step_ms())
        times[name] = float(np.median(ms))
    lo, hi = min(times.values()), max(times.values())
    assert hi / lo < 1.03, times


def test_c5_streams_vs_oracle_lanes(gem):
    """Batched streams: stream s of the GPU == 64-lane oracle lane s (C5 recipe)."""
    S, T = 64, 120
    st = stimulus_streams("c5", 256, T, range(S))
    sim = gem.Simulator(blob("c5"), n_streams=S, flags=gem.GEM_F_DIGEST)
    sim.set_inputs(st)
    sim.step(T)
    po = sim.read_outputs(T)
    dg = sim.read_digests(T)
    o = Oracle(eaig("c5"))
    o.lanes_reset(1)
    r = o.lanes_run(0, st, digest=True)
    assert np.array_equal(po, r["po"])
    assert np.array_equal(dg, r["digest"])


def test_c5_ragged_stream_groups(gem):
    """37 streams (not a multiple of the stream group): every stream matches the oracle lanes."""
    S, T = 37, 60
    st = stimulus_streams("c5", 256, T, range(100, 100 + S))
    sim = gem.Simulator(blob("c5"), n_streams=S, flags=gem.GEM_F_DIGEST)
    assert sim.info["group"] > 1
    sim.set_inputs(st)
    sim.step(T)
    o = Oracle(eaig("c5"))
    o.lanes_reset(1)
    r = o.lanes_run(0, st, digest=True)
    assert np.array_equal(sim.read_outputs(T), r["po"])
    assert np.array_equal(sim.read_digests(T), r["digest"])


@pytest.mark.parametrize("opts,dyn", [("parts=5 stages=2 lanes=1", "1"), ("parts=4 lanes=1", "0"),
                                      ("parts=4 lanes=1", "1"), ("parts=4 lanes=1 lane_m=2", "1"),
                                      ("parts=4 lanes=1 lane_mode=1", "1")])
def test_lane_mode_stages_and_work_distribution(gem, monkeypatch, tmp_path, opts, dyn):
    """Lane mode with two stages (static work lists, cut words between stages)
    and one stage with static (GEM_F_STATIC_LANES) or dynamic ticketed work
    distribution, LAN2 programs with 1 or 2 ops per thread and step, and the
    round-1 boomerang lane programs ("LANE"): 96 streams match the 64-lane
    oracle bit-exactly."""
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    S, T = 96, 50
    net = circuits.small_G(seed=41, n_and=4000, with_ram=True)
    path = circuits.save(net, str(tmp_path), "g")
    b = compile_file(path, opts)
    st = np.stack([stim_random(net.n_pi, T, 2000 + s, reset_pi0_cycles=2) for s in range(S)])
    flags = gem.GEM_F_DIGEST | (gem.GEM_F_STATIC_LANES if dyn == "0" else 0)
    sim = gem.Simulator(b, n_streams=S, flags=flags, grid_limit=3)
    assert sim.info["lanes"] == 1
    sim.set_inputs(st)
    sim.step(T)
    po, dg = sim.read_outputs(T), sim.read_digests(T)
    o = Oracle(path)
    o.lanes_reset(2)
    for g in range(2):
        lo, hi = 64 * g, min(S, 64 * g + 64)
        r = o.lanes_run(g, st[lo:hi], digest=True)
        assert np.array_equal(po[lo:hi], r["po"]), g
        assert np.array_equal(dg[lo:hi], r["digest"]), g


@pytest.mark.parametrize("k", [4, 2])
def test_lane_interleaved_groups_ragged(gem, monkeypatch, tmp_path, k):
    """150 streams = 5 lane groups: work items of K interleaved 32-stream groups
    (one CTA per SM) plus a ragged item; every stream matches the 64-lane
    oracle.  K = 2 on C5, K = 4 on a small design with RAM (C5's lane state is
    too large for 4 groups)."""
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    S, T = 150, 40
    if k == 2:
        path, b, n_pi = eaig("c5"), blob("c5"), 256
        st = stimulus_streams("c5", n_pi, T, range(500, 500 + S))
    else:
        net = circuits.small_G(seed=33, n_and=3000, with_ram=True)
        path = circuits.save(net, str(tmp_path), "g")
        b, n_pi = compile_file(path, "parts=3 lanes=1"), net.n_pi
        st = np.stack([stim_random(n_pi, T, 1000 + s, reset_pi0_cycles=2) for s in range(S)])
    sim = gem.Simulator(b, n_streams=S, flags=gem.GEM_F_DIGEST, lane_ctas_per_sm=1, lane_groups=k)
    assert sim.info["lanes"] == 1 and sim.info["group"] == 32 * k
    sim.set_inputs(st)
    sim.step(T)
    po, dg = sim.read_outputs(T), sim.read_digests(T)
    o = Oracle(path)
    o.lanes_reset(3)
    for g in range(3):
        lo, hi = 64 * g, min(S, 64 * g + 64)
        r = o.lanes_run(g, st[lo:hi], digest=True)
        assert np.array_equal(po[lo:hi], r["po"]), g
        assert np.array_equal(dg[lo:hi], r["digest"]), g


def test_c5_lane_mode_equals_packed_mode(gem, monkeypatch):
    """Stream-sliced lane mode and the bit-packed path give identical traces,
    state and RAMs for the same streams (both checked against the oracle above)."""
    S, T = 40, 50
    st = stimulus_streams("c5", 256, T, range(7, 7 + S))
    lane = gem.Simulator(blob("c5"), n_streams=S)
    assert lane.info["lanes"] == 1
    packed = gem.Simulator(blob("c5"), n_streams=S, flags=gem.GEM_F_NO_LANES)
    assert packed.info["lanes"] == 0
    assert np.array_equal(lane.run(st), packed.run(st))
    assert np.array_equal(lane.read_state(), packed.read_state())
    for s in (0, 33, 39):
        assert np.array_equal(lane.read_ram(1, s), packed.read_ram(1, s))
    q = lane.read_state()
    lane.write_state(q)
    assert np.array_equal(lane.read_state(), q)


@pytest.mark.parametrize("opts,stages", [(None, 1), ("stages=2 levels=10 key=2 part_size=20000", 2)])
def test_c4_sampled_window(gem, opts, stages):
    """C4 (~10M ANDs, 24 RAM blocks) as bench.py maps it (one stage) and with a
    two-stage RepCut mapping: full PO trace and per-cycle flop digests
    for a window the oracle finishes in seconds, plus final state and RAMs."""
    T = 60
    st = stimulus("c4", 512, T)
    sim = gem.Simulator(blob("c4", opts), flags=gem.GEM_F_DIGEST)
    assert sim.info["n_stages"] == stages
    sim.set_inputs(st)
    sim.step(T)
    o = Oracle(eaig("c4"))
    r = o.run(st, digest=True)
    assert np.array_equal(sim.read_outputs(T)[0], r["po"])
    assert np.array_equal(sim.read_digests(T)[0], r["digest"])
    assert np.array_equal(sim.read_state()[0], o.get_state())
    for ram in (0, 17, 23):
        assert np.array_equal(sim.read_ram(ram), o.get_ram(ram))


def test_noinput_and_bad_args(gem):
    sim = gem.Simulator(blob("c1"))
    sim.set_inputs(stimulus("c1", 35, 10))
    with pytest.raises(gem.GemError):
        sim.step(11)
    with pytest.raises(gem.GemError):
        gem.Simulator(b"\0" * 512)


# ------------------------------------------------------------ degenerate cases
def _golden_rows(name):
    import os
    rows = []
    for ln in open(os.path.join(os.path.dirname(__file__), "golden", name)):
        ln = ln.strip()
        if ln and not ln.startswith("#"):
            lhs, rhs = ln.split("|")
            rows.append(([int(x) for x in lhs.split()], [int(x) for x in rhs.split()]))
    return rows


@pytest.mark.parametrize("name", ["half_adder", "toggle", "toggle_init1", "toggle_uninit"])
def test_golden_worked_examples(gem, name):
    """The AIGER-specification worked examples (tests/golden, cited in each
    .expected): a design with no flops (half adder) and designs with no AND
    gate (toggle flop, with reset value 0 and 1) give the printed PO columns,
    for 1 stream and for 3 streams fed the same stimulus."""
    import os
    from gen import pack_bits, unpack_bits
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    p = os.path.join(os.path.dirname(__file__), "golden", name + ".aag")
    rows = _golden_rows(name + ".expected")
    n_pi = len(rows[0][0])
    st = pack_bits(np.array([r[0] for r in rows], np.uint8)) if n_pi else np.zeros((len(rows), 0), np.uint32)
    for opts, ns in [("", 1), ("", 3), ("words=1", 1), ("words=1", 3)]:
        b = compile_file(p, opts)
        sim = gem.Simulator(b, n_streams=ns)
        assert sim.info["words"] == (1 if opts else 0)
        if sim.pi_words:
            sim.set_inputs(np.broadcast_to(st, (ns,) + st.shape))
        else:
            sim.set_inputs(np.zeros((ns, len(rows), 0), np.uint32))
        sim.step(len(rows))
        po = sim.read_outputs(len(rows))
        for s in range(ns):
            assert unpack_bits(po[s], len(rows[0][1])).tolist() == [r[1] for r in rows], (name, ns, s)


def test_wires_constants_and_step0(gem, tmp_path):
    """Degenerate structure: POs that are constants, PIs, inverted PIs and flop
    outputs with no AND gate in between, next to a small random cone; gem_step(0)
    between runs changes neither state nor the following trace."""
    from gen.aig import AigBuilder
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    b = AigBuilder("wires")
    x = b.inputs_n(5)
    q = [b.latch() for _ in range(3)]
    b.set_next(q[0], x[0])
    b.set_next(q[1], q[0] ^ 1)
    b.set_next(q[2], b.AND(x[1], q[1]))
    for lit in (AigBuilder.FALSE, AigBuilder.TRUE, x[2], x[3] ^ 1, q[0], q[1] ^ 1, q[2], b.XOR(x[4], q[2])):
        b.output(lit)
    p = circuits.save(b.finish(), str(tmp_path), "wires")
    st = stim_random(5, 200, 11)
    for opts in ("", "words=1"):
        _wires_run(gem, p, compile_file(p, opts), st, bool(opts))


def _wires_run(gem, p, blob_, st, words):
    sim = gem.Simulator(blob_, flags=gem.GEM_F_TRACE_STATE | gem.GEM_F_DIGEST)
    assert sim.info["words"] == int(words)
    sim.set_inputs(st)
    sim.step(0)
    q0 = sim.read_state()
    sim.step(120)
    po_a = sim.read_outputs(120)
    sim.step(0)
    q1 = sim.read_state()
    sim.step(80)
    po_b = sim.read_outputs(80)
    o = Oracle(p)
    r = o.run(st, state=True)
    assert not q0.any()
    assert np.array_equal(np.concatenate([po_a, po_b], 1)[0], r["po"])
    assert np.array_equal(q1[0], r["state"][119])
    assert np.array_equal(sim.read_state()[0], o.get_state())


# ------------------------------------------------------------ round-2 parity gaps
def test_c3_2000_cycles_ten_checkpoints(gem):
    """C3 as bench.py maps it: 2,000 cycles in 10 steps of 200; full PO trace and
    per-cycle flop digests, and the full flop vector and both RAM blocks at
    each of the 10 checkpoints (SURVEY §8(c) protocol for C3-C5)."""
    T, K = 2000, 10
    st = stimulus("c3", 256, T)
    sim = gem.Simulator(blob("c3"), flags=gem.GEM_F_DIGEST)
    o = Oracle(eaig("c3"))
    for k in range(K):
        a, e = k * T // K, (k + 1) * T // K
        sim.set_inputs(st[a:e])
        sim.step(e - a)
        r = o.run(st[a:e], digest=True)
        assert np.array_equal(sim.read_outputs(e - a)[0], r["po"]), ("PO", k)
        assert np.array_equal(sim.read_digests(e - a)[0], r["digest"]), ("digest", k)
        assert np.array_equal(sim.read_state()[0], o.get_state()), ("state", k)
        for ram in range(o.n_rams):
            assert np.array_equal(sim.read_ram(ram), o.get_ram(ram)), ("ram", k, ram)


def test_c5_bench_size_sampled_shards(gem):
    """C5 in bench.py's launch configuration (4096 streams on one GPU, lane mode
    with 2 or 4 interleaved 32-stream groups per item, >= 4 dynamic work units
    per CTA), 100 cycles: PO trace, per-cycle digests,
    final flops and RAM contents of 1,024 streams = 16 full 64-lane oracle
    groups, covering stream 0, stream 4095 and both sides of every boundary of
    the 2-, 4- and 8-way GPU shards (511|512, 1023|1024, ..., 3583|3584)."""
    S, T = 4096, 100
    sim = gem.Simulator(blob("c5"), n_streams=S, flags=gem.GEM_F_DIGEST)
    info = sim.info
    assert info["lanes"] == 1 and info["group"] in (64, 128)
    items = info["n_parts"] * (S // info["group"])
    assert items >= 4 * info["grid"], (items, info["grid"])   # run = 1: >= 4 dynamic units per CTA
    groups = sorted({0, 63} | {g for b in range(512, 4096, 512) for g in (b // 64 - 1, b // 64)})
    assert len(groups) == 16
    streams = [64 * g + l for g in groups for l in range(64)]
    st_all = np.zeros((S, T, 8), np.uint32)
    st_sel = stimulus_streams("c5", 256, T, streams)
    st_all[streams] = st_sel
    rest = [s for s in range(S) if s not in set(streams)]
    st_all[rest] = stimulus_streams("c5", 256, T, rest[::97])[np.arange(len(rest)) % len(rest[::97])]
    sim.set_inputs(st_all)
    sim.step(T)
    po, dg, q = sim.read_outputs(T), sim.read_digests(T), sim.read_state()
    o = Oracle(eaig("c5"))
    o.lanes_reset(len(groups))
    for j, g in enumerate(groups):
        lo = 64 * g
        r = o.lanes_run(j, st_all[lo:lo + 64], digest=True)
        assert np.array_equal(po[lo:lo + 64], r["po"]), ("PO", g)
        assert np.array_equal(dg[lo:lo + 64], r["digest"]), ("digest", g)
        for lane in range(64):
            assert np.array_equal(q[lo + lane], o.lanes_get_state(j, lane)), ("state", g, lane)
        for lane in (0, 31, 32, 63):
            for ram in range(o.n_rams):
                assert np.array_equal(sim.read_ram(ram, lo + lane), o.lanes_get_ram(j, lane, ram)), (g, lane, ram)


@pytest.mark.parametrize("lanes", [False, True])
def test_ram_preload(gem, tmp_path, lanes):
    """gem_write_ram (RAM preload before the first cycle, include/gem.h; oracle
    side orc_set_ram, pinned in tests/test_oracle.py): random contents per
    block and stream, then 300 cycles; PO/flop trace, final flops and RAM
    contents equal the oracle's, on the bit-packed path (3 streams, two stages)
    and in lane mode (64 streams)."""
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.small_G(seed=21, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    S = 64 if lanes else 3
    T = 300 if not lanes else 120
    rng = np.random.default_rng(77)
    st = np.stack([stim_random(net.n_pi, T, 500 + s, reset_pi0_cycles=2) for s in range(S)])
    b = compile_file(p, "parts=4 lanes=1" if lanes else "parts=4 stages=2")
    sim = gem.Simulator(b, n_streams=S, flags=gem.GEM_F_DIGEST)
    assert sim.info["lanes"] == int(lanes)
    o = Oracle(p)
    assert o.n_rams >= 1
    pre = rng.integers(0, 1 << 32, size=(S, o.n_rams, 8192), dtype=np.uint64).astype(np.uint32)
    for s in range(S):
        for r in range(o.n_rams):
            sim.write_ram(r, pre[s, r], stream=s)
    sim.set_inputs(st)
    sim.step(T)
    po, dg, q = sim.read_outputs(T), sim.read_digests(T), sim.read_state()
    if lanes:
        o.lanes_reset(1)
        for s in range(S):
            for r in range(o.n_rams):
                o.lanes_set_ram(0, s, r, pre[s, r])
        res = o.lanes_run(0, st, digest=True)
        assert np.array_equal(po, res["po"]) and np.array_equal(dg, res["digest"])
        for s in (0, 17, 63):
            assert np.array_equal(q[s], o.lanes_get_state(0, s))
            for r in range(o.n_rams):
                assert np.array_equal(sim.read_ram(r, s), o.lanes_get_ram(0, s, r))
    else:
        for s in range(S):
            os_ = Oracle(p)
            for r in range(o.n_rams):
                os_.set_ram(r, pre[s, r])
            res = os_.run(st[s], digest=True)
            assert np.array_equal(po[s], res["po"]) and np.array_equal(dg[s], res["digest"]), s
            assert np.array_equal(q[s], os_.get_state())
            for r in range(o.n_rams):
                assert np.array_equal(sim.read_ram(r, s), os_.get_ram(r))
    # preloading changes the trace (the RAM data reaches the outputs / flops)
    ref0 = Oracle(p).run(st[0], digest=True)
    assert not np.array_equal(dg[0], ref0["digest"])


def test_uninitialised_latches_read_zero(gem, tmp_path):
    """Reading U5 on a design with many latches: every latch of a random
    sequential design declared uninitialised (AIGER "cur next cur") behaves
    exactly like init 0 on the GPU and in the oracle, and unlike init 1."""
    from gen.aig import write_eaig
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    net = circuits.small_G(seed=5, n_and=2000, with_ram=False, reset=False)
    p0 = circuits.save(net, str(tmp_path), "init0")
    txt = open(p0).read().split("\n")
    hdr = txt[0].split()
    I, L = int(hdr[2]), int(hdr[3])
    def variant(kind):
        lines = list(txt)
        for j in range(L):
            f = lines[1 + I + j].split()
            cur = f[0]
            lines[1 + I + j] = f"{f[0]} {f[1]} " + {"uninit": cur, "one": "1"}[kind]
        q = str(tmp_path / f"{kind}.aag")
        open(q, "w").write("\n".join(lines))
        return q
    pu, p1 = variant("uninit"), variant("one")
    st = stim_random(net.n_pi, 200, 9)
    runs = {}
    for name, p in (("zero", p0), ("uninit", pu), ("one", p1)):
        sim = _full_parity(gem, p, compile_file(p), st)
        runs[name] = sim.read_state()
    assert np.array_equal(runs["zero"], runs["uninit"])
    assert Oracle(pu).get_state().sum() == 0 and Oracle(p1).get_state().any()


def test_single_cta_local_state_resume_and_preload(gem, tmp_path):
    """Single-partition designs run the LOC kernel (flops and RAM-read words kept
    in shared memory across cycles, next cycle's PI words prefetched): state
    written between steps (gem_write_state, checkpoint/resume) and RAM contents
    preloaded with gem_write_ram are picked up by the next launch, and ragged
    steps of 1 cycle work (the prefetch never reads past the queued inputs)."""
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    # C1: resume from a checkpoint taken after 137 cycles, in a fresh simulator
    T = 400
    st = stimulus("c1", 35, T)
    ref = Oracle(eaig("c1")).run(st, state=True)
    a = gem.Simulator(blob("c1"))
    assert a.info["grid"] == 1 and a.info["n_parts"] == 1
    a.set_inputs(st[:137])
    a.step(137)
    q = a.read_state()
    b = gem.Simulator(blob("c1"), flags=gem.GEM_F_TRACE_STATE)
    b.write_state(q)
    po = []
    for a_, e_ in [(137, 138), (138, 139), (139, 250), (250, T)]:
        b.set_inputs(st[a_:e_])
        b.step(e_ - a_)
        po.append(b.read_outputs(e_ - a_)[0])
        assert np.array_equal(b.read_state_trace(e_ - a_)[0], ref["state"][a_:e_])
    assert np.array_equal(np.concatenate(po), ref["po"][137:])
    # a one-partition RAM design: preloaded contents reach the outputs
    p = circuits.save(circuits.ram_direct(), str(tmp_path), "ram")
    o = Oracle(p)
    rng = np.random.default_rng(4)
    pre = rng.integers(0, 1 << 32, 8192, dtype=np.uint64).astype(np.uint32)
    n_pi = o.n_pi
    s2 = rng.integers(0, 1 << 32, size=(200, (n_pi + 31) // 32), dtype=np.uint64).astype(np.uint32)
    s2[:, -1] &= (1 << (n_pi % 32)) - 1 if n_pi % 32 else 0xFFFFFFFF
    sim = gem.Simulator(compile_file(p), flags=gem.GEM_F_DIGEST)
    assert sim.info["grid"] == 1
    sim.write_ram(0, pre)
    o.set_ram(0, pre)
    r = o.run(s2, digest=True)
    sim.set_inputs(s2)
    sim.step(200)
    assert np.array_equal(sim.read_outputs(200)[0], r["po"])
    assert np.array_equal(sim.read_ram(0), o.get_ram(0))
