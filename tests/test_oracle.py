"""Pins for the CPU oracle (tests run without a GPU).

Each test pins the oracle to something other than itself: the AIGER spec's
worked examples (tests/golden), textbook Boolean cells, closed forms (counter,
adder, LFSR period, shift-register delay), a dict model of the RAM readings
U7-U10, invariants (topological order, reset, resume, lanes) and an
independently written Python twin (oracle/twin.py).
"""
import os

import numpy as np
import pytest

from gen import build_c1, pack_bits, stimulus, unpack_bits
from gen.aig import write_eaig
from gen.stimulus import stim_random
from oracle import Oracle, oracle_digest
from oracle.twin import Twin
from tests import circuits

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _num(bits):
    return sum(int(x) << i for i, x in enumerate(bits))


def _read_expected(name):
    rows = []
    for ln in open(os.path.join(GOLD, name)):
        ln = ln.strip()
        if not ln or ln.startswith("#"):
            continue
        lhs, rhs = ln.split("|")
        rows.append(([int(x) for x in lhs.split()], [int(x) for x in rhs.split()]))
    return rows


# ------------------------------------------------------------------ golden
def test_golden_half_adder():
    o = Oracle(os.path.join(GOLD, "half_adder.aag"))
    rows = _read_expected("half_adder.expected")
    stim = pack_bits(np.array([r[0] for r in rows], np.uint8))
    po = unpack_bits(o.run(stim)["po"], 2)
    assert po.tolist() == [r[1] for r in rows]


@pytest.mark.parametrize("name", ["toggle", "toggle_init1", "toggle_uninit"])
def test_golden_toggle(name):
    o = Oracle(os.path.join(GOLD, name + ".aag"))
    rows = _read_expected(name + ".expected")
    stim = np.zeros((len(rows), 0), np.uint32)
    po = unpack_bits(o.run(stim)["po"], 2)
    assert po.tolist() == [r[1] for r in rows]


# ------------------------------------------------------------------ textbook cells
def test_cells_exhaustive(tmp_path):
    p = circuits.save(circuits.cells(), str(tmp_path), "cells")
    o = Oracle(p)
    rows = np.array([[(k >> i) & 1 for i in range(4)] for k in range(16)], np.uint8)
    po = unpack_bits(o.run(pack_bits(rows))["po"], 10)
    for (a, b, c, s), out in zip(rows.tolist(), po.tolist()):
        assert out[0] == a ^ b
        assert out[1] == (a if s else b)
        assert out[2] == int(a + b + c >= 2)
        assert out[3] == (a + b + c) & 1
        assert out[4] == (a + b + c) >> 1
        assert out[5] == 1 - a
        assert out[6] == a & b
        assert out[7] == a | b
        assert out[8] == 0 and out[9] == 1


@pytest.mark.parametrize("seed", range(6))
def test_random_aig_truth_table_vs_twin(tmp_path, seed):
    n_in = 10
    net = circuits.random_comb(n_in, 120, 16, seed)
    p = circuits.save(net, str(tmp_path), f"r{seed}")
    o = Oracle(p)
    rows = np.array([[(k >> i) & 1 for i in range(n_in)] for k in range(1 << n_in)], np.uint8)
    po = unpack_bits(o.run(pack_bits(rows))["po"], 16)
    tpo, _ = Twin(p).run(rows)
    assert np.array_equal(po, tpo)


def test_topological_order_and_renumbering_invariant(tmp_path):
    """Shuffle the ASCII AND lines and permute AND variable ids: same traces."""
    net = circuits.small_G(seed=3, n_and=800, with_ram=True)
    p1 = circuits.save(net, str(tmp_path), "g")
    I, L, A = net.n_inputs, net.n_latches, net.n_ands
    rng = np.random.default_rng(0)
    perm = rng.permutation(A)   # old AND k -> new var id base+perm[k]
    base = I + L + 1

    def m(lit):
        v = int(lit) >> 1
        if v >= base:
            v = base + int(perm[v - base])
        return 2 * v + (int(lit) & 1)

    lines = [f"aag {I + L + A} {I} {L} {net.n_outputs} {A}"]
    lines += [str(2 * (i + 1)) for i in range(I)]
    lines += [f"{2 * (I + 1 + j)} {m(x)}" for j, x in enumerate(net.latch_next)]
    lines += [str(m(x)) for x in net.outputs]
    order = rng.permutation(A)
    lines += [f"{2 * (base + int(perm[k]))} {m(net.and_rhs0[k])} {m(net.and_rhs1[k])}" for k in order]
    lines.append("c")
    for k, r in enumerate(net.rams):
        j = lambda xs: ",".join(str(m(x)) for x in xs)
        lines.append(f"gem-ram {k} rdata={','.join(map(str, r.rdata))} raddr={j(r.raddr)} "
                     f"waddr={j(r.waddr)} wdata={j(r.wdata)} wbe={j(r.wbe)}")
    p2 = os.path.join(str(tmp_path), "g_shuf.aag")
    open(p2, "w").write("\n".join(lines) + "\n")
    o1, o2 = Oracle(p1), Oracle(p2)
    st = stim_random(o1.n_pi, 300, 11, reset_pi0_cycles=2)
    r1 = o1.run(st, state=True)
    r2 = o2.run(st, state=True)
    assert np.array_equal(r1["po"], r2["po"]) and np.array_equal(r1["state"], r2["state"])


def test_binary_and_ascii_agree(tmp_path):
    net = circuits.small_G(seed=5, n_and=1200)
    pa = circuits.save(net, str(tmp_path), "g", binary=False)
    pb = circuits.save(net, str(tmp_path), "g", binary=True)
    st = stim_random(net.n_pi, 200, 1, reset_pi0_cycles=2)
    ra = Oracle(pa).run(st, state=True)
    rb = Oracle(pb).run(st, state=True)
    assert np.array_equal(ra["po"], rb["po"]) and np.array_equal(ra["state"], rb["state"])


# ------------------------------------------------------------------ flops
def test_shift_register_delay(tmp_path):
    k = 7
    o = Oracle(circuits.save(circuits.shift_register(k), str(tmp_path), "sr"))
    rng = np.random.default_rng(4)
    x = rng.integers(0, 2, 200).astype(np.uint8)
    po = unpack_bits(o.run(pack_bits(x[:, None]))["po"], k)
    for j in range(k):
        d = j + 1
        assert np.array_equal(po[d:, j], x[:-d])
        assert not po[:d, j].any()   # init 0 (U5)


# ------------------------------------------------------------------ C1 closed forms
@pytest.fixture(scope="module")
def c1_path(tmp_path_factory):
    d = tmp_path_factory.mktemp("c1")
    p = os.path.join(str(d), "c1.aag")
    write_eaig(build_c1(), p)
    return p


def _c1_fields(po_bits):
    return dict(s=_num(po_bits[0:32]), cout=int(po_bits[32]), cnt=_num(po_bits[33:65]),
                lfsr=_num(po_bits[65:81]), r=_num(po_bits[81:97]))


def test_c1_counter_adder_lfsr_closed_forms(c1_path):
    T = 6000
    o = Oracle(c1_path)
    st = stimulus("c1", 35, T)
    po = unpack_bits(o.run(st)["po"], 97)
    pi = unpack_bits(st, 35)
    rst, en, cin = pi[:, 0], pi[:, 1], pi[:, 2]
    a = np.array([_num(r) for r in pi[:, 3:]], dtype=object)
    cnt = 0
    lfsr = 0
    r = 0
    for t in range(T):
        f = _c1_fields(po[t])
        assert f["cnt"] == cnt, t
        assert f["lfsr"] == lfsr, t
        assert f["r"] == r, t
        tot = cnt + int(a[t]) + int(cin[t])
        assert f["s"] == tot % (1 << 32), t
        assert f["cout"] == tot >> 32, t
        # next state (closed forms of SURVEY §8(c))
        s16 = tot & 0xFFFF
        if rst[t]:
            cnt, lfsr, r = 0, 0xACE1, 0
        else:
            fb = ((lfsr >> 15) ^ (lfsr >> 13) ^ (lfsr >> 12) ^ (lfsr >> 10)) & 1
            r = s16 ^ lfsr
            cnt = (cnt + int(en[t])) % (1 << 32)
            lfsr = ((lfsr << 1) & 0xFFFF) | fb


def test_c1_lfsr_period_65535(c1_path):
    """x^16+x^14+x^13+x^11+1 is primitive: the LFSR period is exactly 65535."""
    o = Oracle(c1_path)
    T = 65535 + 50
    bits = np.zeros((T, 35), np.uint8)
    bits[0, 0] = 1              # one reset cycle -> lfsr = 0xACE1 at t=1
    po = unpack_bits(o.run(pack_bits(bits))["po"], 97)
    lf = np.array([_num(r) for r in po[:, 65:81]])
    assert lf[1] == 0xACE1
    assert np.array_equal(lf[1:41], lf[1 + 65535:41 + 65535])
    first = lf[1:65536]
    assert len(np.unique(first)) == 65535 and 0 not in first


def test_counter_carry_through_all_bits(tmp_path):
    o = Oracle(circuits.save(circuits.counter_with_load(), str(tmp_path), "cl"))
    T = 40
    bits = np.zeros((T, 2), np.uint8)
    bits[0, 0] = 1     # load 0xFFFFFFF0
    bits[1:, 1] = 1    # count every cycle
    po = unpack_bits(o.run(pack_bits(bits))["po"], 32)
    vals = [_num(r) for r in po]
    assert vals[1] == 0xFFFFFFF0
    for t in range(1, T):
        assert vals[t] == (0xFFFFFFF0 + (t - 1)) % (1 << 32)
    assert vals[17] == 0   # carry rippled through all 32 bits


def test_c1_adder_corners(c1_path):
    o = Oracle(c1_path)
    cases = [(0xFFFFFFFF, 1, 0), (0, 0, 0), (0xFFFFFFFF, 0xFFFFFFFF, 1), (0x80000000, 0x80000000, 0),
             (0x12345678, 0x0FEDCBA9, 1)]
    for cnt, a, cin in cases:
        o.reset()
        q = np.zeros(2, np.uint32)
        q[0] = cnt
        o.set_state(q)
        bits = np.zeros((1, 35), np.uint8)
        bits[0, 2] = cin
        bits[0, 3:] = [(a >> i) & 1 for i in range(32)]
        f = _c1_fields(unpack_bits(o.run(pack_bits(bits))["po"], 97)[0])
        tot = cnt + a + cin
        assert f["s"] == tot % (1 << 32) and f["cout"] == tot >> 32


# ------------------------------------------------------------------ RAM readings U7-U10
def test_ram_read_first_dict_model(tmp_path):
    o = Oracle(circuits.save(circuits.ram_direct(), str(tmp_path), "ram"))
    rng = np.random.default_rng(9)
    T = 3000
    ra = rng.integers(0, 16, T)          # small address range -> many collisions
    wa = np.where(rng.random(T) < 0.5, ra, rng.integers(0, 16, T))   # same-address R/W (U8)
    wd = rng.integers(0, 1 << 32, T, dtype=np.uint64)
    be = np.where(rng.random(T) < 0.3, 0xFFFFFFFF, rng.integers(0, 1 << 32, T, dtype=np.uint64))
    be = np.where(rng.random(T) < 0.2, 0, be)
    bits = np.zeros((T, 90), np.uint8)
    for k in range(13):
        bits[:, k] = (ra >> k) & 1
        bits[:, 13 + k] = (wa >> k) & 1
    for k in range(32):
        bits[:, 26 + k] = (wd.astype(np.int64) >> k) & 1
        bits[:, 58 + k] = (be.astype(np.int64) >> k) & 1
    po = unpack_bits(o.run(pack_bits(bits))["po"], 32)
    mem = {}
    rd = 0                                 # U10: registered read data starts at 0
    n_same = 0
    for t in range(T):
        assert _num(po[t]) == rd, t        # U7: value read at t-1 is visible at t
        new_rd = mem.get(int(ra[t]), 0)    # U8: read before the write
        m = int(be[t])
        mem[int(wa[t])] = (mem.get(int(wa[t]), 0) & ~m & 0xFFFFFFFF) | (int(wd[t]) & m)   # U9
        n_same += int(ra[t] == wa[t] and m != 0)
        rd = new_rd
    assert n_same > 100
    # the RAM contents are readable and equal the model
    ram = o.get_ram(0)
    for a_, v in mem.items():
        assert ram[a_] == v


def test_ram_write_then_read_latency(tmp_path):
    """Write k@a at t, read a at t+1 -> visible on rdata at t+2."""
    o = Oracle(circuits.save(circuits.ram_direct(), str(tmp_path), "ram"))
    T = 4
    bits = np.zeros((T, 90), np.uint8)
    a, k = 0x155, 0xDEADBEEF
    for i in range(13):
        bits[0, 13 + i] = (a >> i) & 1     # waddr at t=0
        bits[1, i] = (a >> i) & 1          # raddr at t=1
    for i in range(32):
        bits[0, 26 + i] = (k >> i) & 1
        bits[0, 58 + i] = 1
    po = unpack_bits(o.run(pack_bits(bits))["po"], 32)
    assert [_num(r) for r in po] == [0, 0, k, 0]


def test_ram_preload_dict_model(tmp_path):
    """orc_set_ram (the oracle side of gem_write_ram): a block preloaded with
    random contents is read first-then-written exactly like the dict model of
    test_ram_read_first_dict_model started from those contents (U7-U10); the
    64-lane variant with per-lane preloads gives every lane its own model."""
    p = circuits.save(circuits.ram_direct(), str(tmp_path), "ram")
    rng = np.random.default_rng(19)
    T = 400
    init = rng.integers(0, 1 << 32, 8192, dtype=np.uint64).astype(np.uint32)
    ra = rng.integers(0, 64, T)
    wa = np.where(rng.random(T) < 0.5, ra, rng.integers(0, 64, T))
    wd = rng.integers(0, 1 << 32, T, dtype=np.uint64)
    be = np.where(rng.random(T) < 0.4, 0, rng.integers(0, 1 << 32, T, dtype=np.uint64))
    bits = np.zeros((T, 90), np.uint8)
    for k in range(13):
        bits[:, k] = (ra >> k) & 1
        bits[:, 13 + k] = (wa >> k) & 1
    for k in range(32):
        bits[:, 26 + k] = (wd.astype(np.int64) >> k) & 1
        bits[:, 58 + k] = (be.astype(np.int64) >> k) & 1
    stim = pack_bits(bits)

    def model(mem0):
        mem = {a_: int(mem0[a_]) for a_ in range(8192)}
        rd, out = 0, []
        for t in range(T):
            out.append(rd)
            new_rd = mem[int(ra[t])]
            m = int(be[t])
            mem[int(wa[t])] = (mem[int(wa[t])] & ~m & 0xFFFFFFFF) | (int(wd[t]) & m)
            rd = new_rd
        return out, np.array([mem[a_] for a_ in range(8192)], np.uint32)

    exp_po, exp_mem = model(init)
    o = Oracle(p)
    o.set_ram(0, init)
    po = unpack_bits(o.run(stim)["po"], 32)
    assert [_num(r) for r in po] == exp_po
    assert np.array_equal(o.get_ram(0), exp_mem)
    # 64-lane group: lane l preloaded with init ^ l, same port traffic
    o.lanes_reset(1)
    for lane in (0, 5, 63):
        o.lanes_set_ram(0, lane, 0, init ^ np.uint32(lane))
    r = o.lanes_run(0, np.broadcast_to(stim, (64,) + stim.shape))
    for lane in (0, 5, 63):
        e_po, e_mem = model(init ^ np.uint32(lane))
        assert [_num(x) for x in unpack_bits(r["po"][lane], 32)] == e_po, lane
        assert np.array_equal(o.lanes_get_ram(0, lane, 0), e_mem), lane
    e_po0, _ = model(np.zeros(8192, np.uint32))
    assert [_num(x) for x in unpack_bits(r["po"][1], 32)] == e_po0   # not preloaded: U10 zeros


# ------------------------------------------------------------------ invariants
def test_reset_makes_state_independent_of_prefix(tmp_path):
    net = circuits.small_G(seed=11, n_and=2000, with_ram=False, reset=True)
    p = circuits.save(net, str(tmp_path), "g")
    R = 1
    finals = []
    for seed in (1, 2, 3):
        o = Oracle(p)
        pre = stim_random(net.n_pi, 50, seed)
        o.run(pre)
        rst = stim_random(net.n_pi, R, 100 + seed, reset_pi0_cycles=R)
        o.run(rst)
        finals.append(o.get_state())
    assert np.array_equal(finals[0], finals[1]) and np.array_equal(finals[0], finals[2])
    assert not finals[0].any()    # every flop D is gated by !rst


def test_resume_and_state_roundtrip(tmp_path):
    net = circuits.small_G(seed=13, n_and=2000)
    p = circuits.save(net, str(tmp_path), "g")
    st = stim_random(net.n_pi, 400, 5, reset_pi0_cycles=3)
    a = Oracle(p)
    ra = a.run(st, state=True)
    b = Oracle(p)
    rb1 = b.run(st[:150], state=True)
    rb2 = b.run(st[150:], state=True)
    assert np.array_equal(ra["po"], np.concatenate([rb1["po"], rb2["po"]]))
    assert np.array_equal(ra["state"], np.concatenate([rb1["state"], rb2["state"]]))
    # get/set state round trip reproduces the continuation (no RAM: Q is the whole state)
    net2 = circuits.small_G(seed=14, n_and=2000, with_ram=False)
    p2 = circuits.save(net2, str(tmp_path), "g2")
    st2 = stim_random(net2.n_pi, 300, 6, reset_pi0_cycles=3)
    c = Oracle(p2)
    c.run(st2[:150])
    q = c.get_state()
    d = Oracle(p2)
    d.set_state(q)
    assert np.array_equal(d.get_state(), q)
    rc = c.run(st2[150:], state=True)
    rd = d.run(st2[150:], state=True)
    assert np.array_equal(rc["po"], rd["po"]) and np.array_equal(rc["state"], rd["state"])


def test_twin_agrees_on_sequential_prefix(tmp_path):
    net = circuits.small_G(seed=17, n_and=1500)
    p = circuits.save(net, str(tmp_path), "g")
    st = stim_random(net.n_pi, 60, 3, reset_pi0_cycles=2)
    r = Oracle(p).run(st, state=True)
    tpo, tq = Twin(p).run(unpack_bits(st, net.n_pi))
    assert np.array_equal(r["po"], pack_bits(tpo))
    assert np.array_equal(r["state"], pack_bits(tq))


def test_lanes_equal_single_stream(tmp_path):
    net = circuits.small_G(seed=19, n_and=1500)
    p = circuits.save(net, str(tmp_path), "g")
    lanes = 37
    T = 80
    stims = np.stack([stim_random(net.n_pi, T, 1000 + s, reset_pi0_cycles=2) for s in range(lanes)])
    o = Oracle(p)
    o.lanes_reset(1)
    rl = o.lanes_run(0, stims, digest=True)
    for s in (0, 5, 36):
        single = Oracle(p)
        rs = single.run(stims[s], digest=True)
        assert np.array_equal(rl["po"][s], rs["po"])
        assert np.array_equal(rl["digest"][s], rs["digest"])
        assert np.array_equal(o.lanes_get_state(0, s), single.get_state())


# ------------------------------------------------------------------ digest spec
def test_digest_closed_form():
    # d = sum_w rotl64(word_w, w mod 64) * (2w+1)
    assert oracle_digest(np.array([1], np.uint32)) == 1
    assert oracle_digest(np.array([1, 1], np.uint32)) == 1 + 2 * 3
    assert oracle_digest(np.array([0, 0, 0x80000000], np.uint32)) == (0x80000000 << 2) * 5
    w = np.zeros(66, np.uint32)
    w[65] = 0xFFFFFFFF     # rotation index 65 mod 64 = 1
    assert oracle_digest(w) == ((0xFFFFFFFF << 1) * 131) % (1 << 64)
    w = np.zeros(64, np.uint32)
    w[63] = 3              # rotl by 63: bit0 -> bit63, bit1 -> bit0
    assert oracle_digest(w) == (((1 << 63) | 1) * 127) % (1 << 64)


def test_state_trace_digest_consistency(c1_path):
    o = Oracle(c1_path)
    r = o.run(stimulus("c1", 35, 100), state=True, digest=True)
    for t in range(100):
        assert r["digest"][t] == oracle_digest(r["state"][t])


# ------------------------------------------------------------------ parser rejects
@pytest.mark.parametrize("text,msg", [
    ("aag 3 1 0 1 2\n2\n6\n4 6 2\n6 4 2\n", "loop"),
    ("aag 1 1 0 0 0 1\n2\n", "B/C/J/F"),
    ("aig 1 1 0 0 0\n", "AND"),
    ("aag 2 1 0 1 1\n2\n4\n4 2 9\n", "range"),
])
def test_parser_rejects(tmp_path, text, msg):
    p = os.path.join(str(tmp_path), "bad.aag")
    open(p, "w").write(text)
    if msg == "AND":
        Oracle(p)   # header-only binary file with 0 ANDs is fine
        return
    with pytest.raises(ValueError):
        Oracle(p)


def test_parser_rejects_double_owned_rdata(tmp_path):
    net = circuits.ram_direct()
    p = circuits.save(net, str(tmp_path), "ram")
    txt = open(p).read()
    line = [ln for ln in txt.splitlines() if ln.startswith("gem-ram")][0]
    open(p, "w").write(txt + line.replace("gem-ram 0", "gem-ram 1") + "\n")
    with pytest.raises(ValueError):
        Oracle(p)


def test_gated_counters_closed_form(tmp_path):
    """Closed form for the activity-pruning test design (tests/circuits.py
    gated_counters): counter k at cycle t = number of cycles u < t with en_k(u)=1,
    mod 2^16 (flop semantics: 1-cycle delay, PO sampled before the edge, U11)."""
    from gen.stimulus import stim_bursts
    net = circuits.gated_counters(8, 16)
    p = circuits.save(net, str(tmp_path), "gated")
    st = stim_bursts(8, 700, 11)
    po = Oracle(p).run(st)["po"].astype(np.int64)
    en = st[:, 0].astype(np.int64)
    for k in range(8):
        want = np.concatenate([[0], np.cumsum((en >> k) & 1)[:-1]]) & 0xFFFF
        got = (po[:, k] & 0xFFFF)          # module k's POs: cnt (16 bits) then acc (16 bits) = word k
        assert np.array_equal(got, want), k
        on = ((en >> k) & 1).astype(bool)
        acc = po[:, k] >> 16               # acc only changes in cycles after an enabled one
        assert np.array_equal(acc[1:][~on[:-1]], acc[:-1][~on[:-1]]), k


@pytest.mark.parametrize("threads", [1, 3, 8])
def test_level_parallel_variant_equals_oracle(tmp_path, threads):
    """The level-parallel CPU baseline (SURVEY §8(d) nproc-thread variant) gives
    the oracle's PO trace and final state on a design with RAM, resets and
    long tails (small levels evaluated serially, wide ones split)."""
    net = circuits.small_G(seed=21, n_and=20000, with_ram=True, clusters=4, flops=256, d_max=40)
    p = circuits.save(net, str(tmp_path), "g")
    st = stim_random(net.n_pi, 300, 5, reset_pi0_cycles=2)
    a = Oracle(p)
    ref = a.run(st)["po"]
    b = Oracle(p)
    got = b.run_mt(st, threads)
    assert np.array_equal(got, ref)
    assert np.array_equal(b.get_state(), a.get_state())
    for r in range(len(net.rams)):
        assert np.array_equal(b.get_ram(r), a.get_ram(r))
