"""Small hand-built test circuits (INPUT side: structure only, no evaluation)."""
from __future__ import annotations

import os

import numpy as np

from gen.aig import AigBuilder, Netlist, write_eaig
from gen.netlists import ClusterSpec, GSpec, RamMacroSpec, build_G


def save(net: Netlist, d: str, name: str, binary=False) -> str:
    p = os.path.join(d, name + (".aig" if binary else ".aag"))
    write_eaig(net, p, binary=binary)
    return p


def cells() -> Netlist:
    """PIs a b c s; POs: a^b, s?a:b, maj(a,b,c), fa.sum, fa.cout, !a, a&b, a|b, const0, const1."""
    b = AigBuilder("cells")
    a, bb, c, s = b.inputs_n(4)
    b.output(b.XOR(a, bb))
    b.output(b.MUX(s, a, bb))
    b.output(b.MAJ(a, bb, c))
    fs, fc = b.full_adder(a, bb, c)
    b.output(fs)
    b.output(fc)
    b.output(b.NOT(a))
    b.output(b.AND(a, bb))
    b.output(b.OR(a, bb))
    b.output(AigBuilder.FALSE)
    b.output(AigBuilder.TRUE)
    return b.finish()


def random_comb(n_in: int, n_and: int, n_out: int, seed: int) -> Netlist:
    rng = np.random.default_rng(seed)
    b = AigBuilder(f"rand{seed}")
    lits = b.inputs_n(n_in)
    for _ in range(n_and):
        x = lits[rng.integers(len(lits))] ^ int(rng.integers(2))
        y = lits[rng.integers(len(lits))] ^ int(rng.integers(2))
        lits.append(b.AND(x, y))
    for k in range(n_out):
        b.output(lits[-1 - k] ^ int(rng.integers(2)))
    return b.finish()


def shift_register(k: int) -> Netlist:
    """1 PI -> k flops in a chain; POs = every flop (PO j = PI delayed by j+1)."""
    b = AigBuilder(f"shift{k}")
    x = b.input()
    prev = x
    fl = []
    for _ in range(k):
        q = b.latch()
        b.set_next(q, prev)
        fl.append(q)
        prev = q
    for q in fl:
        b.output(q)
    return b.finish()


def counter_with_load(width: int = 32, preset: int = 0xFFFFFFF0) -> Netlist:
    """PIs: load, en.  cnt' = load ? preset : cnt + en.  POs: cnt."""
    b = AigBuilder("cntload")
    load, en = b.input(), b.input()
    cnt = [b.latch() for _ in range(width)]
    carry = en
    for i in range(width):
        s = b.XOR(cnt[i], carry)
        carry = b.AND(cnt[i], carry)
        pv = AigBuilder.TRUE if (preset >> i) & 1 else AigBuilder.FALSE
        b.set_next(cnt[i], b.MUX(load, pv, s))
    for q in cnt:
        b.output(q)
    return b.finish()


def ram_direct(seed: int = 0) -> Netlist:
    """One RAM block whose ports are PIs: raddr(13) waddr(13) wdata(32) wbe(32) = 90 PIs.

    POs = the 32 rdata bits.  A same-address pin needs waddr == raddr often,
    which the stimulus controls.
    """
    b = AigBuilder("ramdirect")
    ra = b.inputs_n(13)
    wa = b.inputs_n(13)
    wd = b.inputs_n(32)
    be = b.inputs_n(32)
    rd = b.ram(ra, wa, wd, be)
    for x in rd:
        b.output(x)
    return b.finish()


def small_G(seed: int = 7, n_and: int = 3000, with_ram: bool = True, reset: bool = True,
            clusters: int = 4, flops: int = 256, d_max: int = 24, tail: bool = True) -> Netlist:
    cl = []
    for c in range(clusters):
        t = 8 if (tail and c == 0) else 0
        cl.append(ClusterSpec(n_and=n_and // clusters, n_flop=flops // clusters,
                              d_max=d_max if t else min(d_max, 16), tau=4.0, n_tail=t,
                              d_head=12 if t else 0))
    rams = [RamMacroSpec(owner=1, readers=[1, 2])] if with_ram else []
    spec = GSpec("smallG", cl, n_pi=40, n_po=40, p_x=0.05, rams=rams, reset_pi0=reset,
                 pi_per_cluster=8, neighbour_flops=16)
    net, _ = build_G(spec, seed)
    return net


def gated_counters(n_blocks: int = 8, width: int = 16) -> Netlist:
    """n_blocks independent modules with their own enable PI: cnt_k' = cnt_k + en_k,
    acc_k' = acc_k ^ (cnt_k ^ (cnt_k << 1)) when en_k (a module that is idle while
    its enable is 0).  PIs: en_0..en_{n-1}; POs: every cnt/acc bit.  Used by the
    activity-pruning tests (row f3): idle modules' partitions see unchanged inputs."""
    b = AigBuilder(f"gated{n_blocks}x{width}")
    ens = b.inputs_n(n_blocks)
    for k in range(n_blocks):
        en = ens[k]
        cnt = [b.latch() for _ in range(width)]
        acc = [b.latch(init=(k + i) & 1) for i in range(width)]
        carry = en
        for i in range(width):
            b.set_next(cnt[i], b.XOR(cnt[i], carry))
            carry = b.AND(cnt[i], carry)
        for i in range(width):
            mix = b.XOR(cnt[i], cnt[i - 1] if i else AigBuilder.FALSE)
            b.set_next(acc[i], b.MUX(en, b.XOR(acc[i], mix), acc[i]))
        for q in cnt + acc:
            b.output(q)
    return b.finish()


def gated_modules(n_blocks: int = 64, flops: int = 64, width: int = 256, depth: int = 48, seed: int = 1) -> Netlist:
    """n_blocks modules of random layered logic (depth `depth`, `width` ANDs per
    level over the module's own flops) whose flops load the logic's outputs only
    while the module's enable PI is 1 (q' = en ? f(q) : q).  PIs: en_k; POs: the
    first 8 flops of each module.  The measurement design of row f3."""
    rng = np.random.default_rng(seed)
    b = AigBuilder(f"gmods{n_blocks}")
    ens = b.inputs_n(n_blocks)
    for k in range(n_blocks):
        q = [b.latch(init=int(rng.integers(2))) for _ in range(flops)]
        levels = [q]
        for _ in range(depth):
            prev = levels[-1]
            pool = [x for lv in levels[-3:] for x in lv]
            cur = []
            for _ in range(width):
                x = prev[int(rng.integers(len(prev)))] ^ int(rng.integers(2))
                y = pool[int(rng.integers(len(pool)))] ^ int(rng.integers(2))
                cur.append(b.AND(x, y))
            levels.append(cur)
        last = levels[-1]
        for i in range(flops):
            b.set_next(q[i], b.MUX(ens[k], last[i % len(last)] ^ (i & 1), q[i]))
        for i in range(8):
            b.output(q[i])
    return b.finish()


def deep_chains(width: int = 64, chain: int = 120, seed: int = 3) -> Netlist:
    """Depth-synthesis workload (gem_synth.h): a `width`-bit ripple-carry
    adder of two PIs words plus a flop word (majority-cell carry chain), a
    `width`-bit incrementer of a flop word (AND chain), a `chain`-long
    AND/OR priority chain with random edge inversions (single-AND links), and
    a linear 48-input AND (a balancing supergate).  POs: every sum bit, the
    carry out, every priority-chain node, the wide AND."""
    rng = np.random.default_rng(seed)
    b = AigBuilder(f"chains{seed}")
    x = b.inputs_n(width)
    y = b.inputs_n(width)
    en = b.input()
    q = [b.latch() for _ in range(width)]
    r = [b.latch() for _ in range(width)]
    c = en
    for i in range(width):                        # r' = r + 1 (when en): incrementer
        b.set_next(r[i], b.XOR(r[i], c))
        c = b.AND(r[i], c)
    c = b.AND(x[0], en)
    for i in range(width):                        # s = x + y + q: two ripple adders
        t, c1 = b.full_adder(x[i], y[i], c)
        s, c = b.full_adder(t, q[i], c1)
        b.output(s)
        b.set_next(q[i], s)
    b.output(c)
    side = b.inputs_n(16)
    n = side[0]
    for k in range(chain):                        # alternating AND/OR priority chain
        n = b.AND(n ^ int(rng.integers(0, 2)), side[int(rng.integers(0, 16))] ^ int(rng.integers(0, 2)))
        b.output(n)
    a = x[0]
    for i in range(1, 48):
        a = b.AND(a, y[i % width])
    b.output(a)
    return b.finish()
