"""Mapper + bitstream checks on CPU: the CPU ISA interpreter (tests/isa, a test
tool executing the ISA definition) must reproduce the oracle exactly, so mapper
bugs are caught without a GPU.  Metamorphic: partition count, stage count and
the leaf cap must not change results."""
import os

import numpy as np
import pytest

from gen import build_c1, stimulus
from gen.aig import write_eaig
from gen.stimulus import stim_random
from oracle import Oracle
from paper_conf_dac_guozwlr25_b200.isa import blob_info
from paper_conf_dac_guozwlr25_b200.mapping import compile_file
from tests import circuits
from tests.common import blob, eaig
from tests.isa import IsaInterp


def _check(path, b, stim):
    r = Oracle(path).run(stim, state=True)
    po, q = IsaInterp(b).run(stim)
    assert np.array_equal(po, r["po"]), np.where((po != r["po"]).any(1))[0][:5]
    assert np.array_equal(q, r["state"]), np.where((q != r["state"]).any(1))[0][:5]


def test_c1_isa_matches_oracle(tmp_path):
    p = os.path.join(str(tmp_path), "c1.aag")
    write_eaig(build_c1(), p)
    b = compile_file(p)
    info = blob_info(b)
    assert info.n_parts == 1 and info.n_and > 500
    _check(p, b, stimulus("c1", 35, 3000))


@pytest.mark.parametrize("opts", ["parts=1", "parts=3", "parts=6 leafcap=64", "parts=5 stages=2",
                                  "parts=4 stages=2 cut_level=3", "parts=2 max_state_words=256"])
def test_small_designs_metamorphic(tmp_path, opts):
    net = circuits.small_G(seed=21, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    b = compile_file(p, opts)
    _check(p, b, stim_random(net.n_pi, 150, 3, reset_pi0_cycles=2))


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_random_comb_and_cells(tmp_path, seed):
    for name, net in [("rc", circuits.random_comb(12, 300, 20, seed)), ("cells", circuits.cells()),
                      ("sr", circuits.shift_register(40)), ("ram", circuits.ram_direct()),
                      ("cnt", circuits.counter_with_load())]:
        p = circuits.save(net, str(tmp_path), name)
        b = compile_file(p)
        rng = np.random.default_rng(seed)
        n_pi = Oracle(p).n_pi
        st = rng.integers(0, 1 << 32, size=(200, (n_pi + 31) // 32), dtype=np.uint64).astype(np.uint32)
        if n_pi % 32:
            st[:, -1] &= (1 << (n_pi % 32)) - 1
        if name == "ram":   # force same-address traffic
            st[:, 0] = (st[:, 0] & ~np.uint32(0x3FFFFFF)) | (st[:, 0] & 0x7) | ((st[:, 0] & 0x7) << 13)
        _check(p, b, st)


@pytest.mark.parametrize("synth", [0, 1, 2])
def test_depth_synthesis_preserves_function(tmp_path, synth):
    """Depth-oriented synthesis (gem_synth.h: AND balancing, chain
    lookahead) is an identity of Boolean algebra: the mapped program of every
    synthesis level reproduces the oracle, which runs the ORIGINAL netlist."""
    net = circuits.deep_chains(48, 90, seed=synth + 5)
    p = circuits.save(net, str(tmp_path), "chains")
    b = compile_file(p, f"synth={synth} parts=2")
    n_pi = Oracle(p).n_pi
    rng = np.random.default_rng(synth)
    st = rng.integers(0, 1 << 32, size=(300, (n_pi + 31) // 32), dtype=np.uint64).astype(np.uint32)
    st[:, -1] &= (1 << (n_pi % 32)) - 1
    _check(p, b, st)


def test_depth_synthesis_reduces_levels(tmp_path):
    """Chains of length n go from O(n) to O(log n) levels: a 64-bit two-adder
    carry chain (majority cells), a 64-bit incrementer and a 200-link AND/OR
    priority chain (depth >= 128 before) end below 40 levels; balancing alone
    turns the 48-input linear AND into a tree; the live AND count is the
    pre-synthesis one (reading U14) and the synthesised one is reported."""
    net = circuits.deep_chains(64, 200, seed=1)
    p = circuits.save(net, str(tmp_path), "chains")
    i0 = blob_info(compile_file(p, "synth=0"))
    i1 = blob_info(compile_file(p, "synth=1"))
    i2 = blob_info(compile_file(p, "synth=2"))
    assert i0.max_levels == i0.levels_in >= 200
    assert i1.levels_in == i0.levels_in and i2.levels_in == i0.levels_in
    assert i2.max_levels <= 40 and i2.synth_chains >= 3, (i2.max_levels, i2.synth_chains)
    assert i2.max_layers < i0.max_layers
    assert i0.n_and == i1.n_and == i2.n_and and i2.n_and_synth > i0.n_and
    assert i1.synth_chains == 0 and i1.n_and_synth <= i0.n_and


def test_c3_synthesis_depth():
    """BASELINE config 3's deep long-tailed paths (carry-chain tails):
    synthesis cuts the logic depth by > 2x and the critical layers with it."""
    i = blob_info(blob("c3"))
    assert i.levels_in == 129 and i.max_levels <= 64, (i.levels_in, i.max_levels)
    assert sum(i.stage_max_layers()) <= 10
    assert i.synth_growth < 0.10


def test_km1_refinement_reduces_replication_for_any_order(tmp_path):
    """Partitioning: the k-way min-cut refinement of
    the RepCut hypergraph lowers replication (Σ partition cones / live ANDs - 1)
    well below what greedy packing reaches, whatever endpoint order the packing
    starts from (register declaration order, smallest register read, deep-cone
    min-hash), and the refined mappings stay bit-exact."""
    net = circuits.small_G(seed=3, n_and=12000, with_ram=True, clusters=8, flops=512)
    p = circuits.save(net, str(tmp_path), "g8")
    st = stim_random(net.n_pi, 60, 7, reset_pi0_cycles=2)
    reps = {}
    for key in (0, 1, 2):
        base = f"parts=8 merge=0 refine=0 key={key} km1_pins=100000"
        r0 = blob_info(compile_file(p, base + " km1=0")).replication
        b = compile_file(p, base)
        r1 = blob_info(b).replication
        assert r1 < 0.7 * r0, (key, r0, r1)
        reps[key] = r1
        _check(p, b, st)
    assert max(reps.values()) < 2.0 * min(reps.values()), reps


def test_c2_prefix():
    _check(eaig("c2"), blob("c2"), stimulus("c2", 128, 120))


@pytest.mark.slow
def test_c3_prefix():
    _check(eaig("c3"), blob("c3"), stimulus("c3", 256, 12))


def test_blob_stats_c2():
    i = blob_info(blob("c2"))
    assert i.n_and > 90_000
    assert i.max_layers >= 40 / 13          # cannot beat 13 levels per layer
    assert i.max_layers <= 40               # boomerang layers are fewer than levels
    assert i.max_state_words <= 2048
    # part table decoded with the header's stride: per-part layer counts add up
    assert sum(i.part_layers) == i.total_layers
    assert max(i.part_layers) == i.max_layers
    assert all(c > 0 for c in i.part_cost)


@pytest.mark.parametrize("opts", ["parts=1 lanes=1", "parts=4 lanes=1", "parts=5 stages=2 lanes=1"])
def test_lane_programs_match_oracle_lanes(tmp_path, opts):
    """Lane-mode programs (32 streams per lane word) through the CPU ISA
    interpreter == the oracle's 64-lane batched mode, stream by stream."""
    net = circuits.small_G(seed=23, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    b = compile_file(p, opts)
    st = np.stack([stim_random(net.n_pi, 80, 500 + s, reset_pi0_cycles=2) for s in range(32)])
    po, q = IsaInterp(b).run_lanes(st)
    o = Oracle(p)
    o.lanes_reset(1)
    r = o.lanes_run(0, st)
    assert np.array_equal(po, r["po"])


def test_c5_lane_program_prefix():
    from gen import stimulus_streams
    st = stimulus_streams("c5", 256, 6, range(32))
    po, q = IsaInterp(blob("c5")).run_lanes(st)
    o = Oracle(eaig("c5"))
    o.lanes_reset(1)
    r = o.lanes_run(0, st)
    assert np.array_equal(po, r["po"])


def _lane_programs(b):
    """(partition id, lane program words) for every partition of a blob."""
    w = np.frombuffer(b, np.uint32)
    n_parts, off_parts, off_lane = int(w[6]), int(w[21]), int(w[37])
    for p in range(n_parts):
        pt = w[off_parts + 16 * p: off_parts + 16 * p + 16]
        yield p, w[off_lane + int(pt[9]): off_lane + int(pt[9]) + int(pt[10])]


def test_lane_layer_headers_carry_next_layer():
    """gem_isa.h LLH_NEXT: layer l's header words [16, 28) equal layer l+1's
    words [0, 12) (zeros after the last layer) -- the kernel issues layer l+1's
    record loads from them without reading its header first."""
    LPH_N_LAYERS, LPH_OFF_LAYERS = 2, 7
    n_checked = 0
    from tests.common import MAP_OPTS
    for _, pr in _lane_programs(blob("c5", MAP_OPTS["c5"] + " lane_mode=1")):
        L = int(pr[LPH_OFF_LAYERS])
        for l in range(int(pr[LPH_N_LAYERS])):
            nxt = L + int(pr[L])
            want = pr[nxt:nxt + 12] if l + 1 < int(pr[LPH_N_LAYERS]) else np.zeros(12, np.uint32)
            assert np.array_equal(pr[L + 16:L + 28], want), l
            L = nxt
            n_checked += 1
    assert n_checked > 100


def test_program_tail_holds_gread_used_bit_masks(tmp_path):
    """Row f3 (GEM_F_ACTIVITY): the last ceil4(n_gread) words of a partition
    program are the used-bit masks of its gread words: every mask is non-zero,
    and together they cover exactly the sources the partition reads."""
    net = circuits.gated_counters(8, 16)
    p = circuits.save(net, str(tmp_path), "gated")
    b = compile_file(p, "parts=8")
    w = np.frombuffer(b, np.uint32)
    n_parts, off_parts, off_prog = int(w[6]), int(w[21]), int(w[24])
    total_bits = 0
    for q in range(n_parts):
        pt = w[off_parts + 16 * q: off_parts + 16 * q + 16]
        pr = w[off_prog + int(pt[1]): off_prog + int(pt[1]) + int(pt[2])]
        n_gread = int(pr[1])
        masks = pr[len(pr) - ((n_gread + 3) & ~3):][:n_gread]
        assert n_gread > 0 and (masks != 0).all()
        total_bits += sum(bin(int(m)).count("1") for m in masks)
    # each module reads its enable and its 32 flops: 8 partitions x 33 sources
    assert total_bits == 8 * 33, total_bits


# ---------------------------------------------------------------- word programs (WRD1)
def _check_words(path, b, stim):
    assert blob_info(b).has_words, "mapper emitted no word programs"
    r = Oracle(path).run(stim, state=True)
    po, q = IsaInterp(b).run(stim, words=True)
    assert np.array_equal(po, r["po"]), np.where((po != r["po"]).any(1))[0][:5]
    assert np.array_equal(q, r["state"]), np.where((q != r["state"]).any(1))[0][:5]


def test_c1_word_program_matches_oracle(tmp_path):
    p = os.path.join(str(tmp_path), "c1.aag")
    write_eaig(build_c1(), p)
    b = compile_file(p, "levels=10 words=1")
    info = blob_info(b)
    # depth-bound: one step per level of the synthesised C1 (20 levels)
    assert info.word_max_steps == info.max_levels
    _check_words(p, b, stimulus("c1", 35, 3000))


@pytest.mark.parametrize("opts", ["parts=1", "parts=3 word_step=64", "parts=5 stages=2", "parts=4 stages=2 cut_level=3",
                                  "parts=2 word_step=32"])
def test_small_designs_word_programs(tmp_path, opts):
    net = circuits.small_G(seed=21, n_and=4000, with_ram=True)
    p = circuits.save(net, str(tmp_path), "g")
    b = compile_file(p, opts + " words=1")
    _check_words(p, b, stim_random(net.n_pi, 150, 3, reset_pi0_cycles=2))


@pytest.mark.parametrize("seed", [1, 2])
def test_word_programs_cells(tmp_path, seed):
    for name, net in [("rc", circuits.random_comb(12, 300, 20, seed)), ("cells", circuits.cells()),
                      ("sr", circuits.shift_register(40)), ("ram", circuits.ram_direct()),
                      ("cnt", circuits.counter_with_load())]:
        p = circuits.save(net, str(tmp_path), name)
        b = compile_file(p, "words=1")
        rng = np.random.default_rng(seed)
        n_pi = Oracle(p).n_pi
        st = rng.integers(0, 1 << 32, size=(200, (n_pi + 31) // 32), dtype=np.uint64).astype(np.uint32)
        if n_pi % 32:
            st[:, -1] &= (1 << (n_pi % 32)) - 1
        if name == "ram":
            st[:, 0] = (st[:, 0] & ~np.uint32(0x3FFFFFF)) | (st[:, 0] & 0x7) | ((st[:, 0] & 0x7) << 13)
        _check_words(p, b, st)


def test_c2_word_program_prefix(tmp_path):
    from tests.common import MAP_OPTS
    b = blob("c2", MAP_OPTS["c2"] + " words=1")
    info = blob_info(b)
    assert info.word_max_steps <= info.max_levels + 1
    _check_words(eaig("c2"), b, stimulus("c2", 128, 60))
