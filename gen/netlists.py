"""Seeded synthetic netlist generators for configs C1..C5 (INPUT side only).

Shapes follow SURVEY.md §8(d) (themselves derived from PAPER.md Table I,
P:186-194, and Observation 4: "a large portion of the gates reside in a
few frontier levels whereas only a few gates are accountable for the rest").

  C1  32-bit counter + 32-bit ripple-carry adder + 16-bit LFSR (hand-built).
  C2  cluster-structured levelised random AIG, ~100K ANDs, 4K flops, depth 40.
  C3  CPU-core-shaped, ~1M ANDs, 32K flops, 2 RAM blocks (64 KiB), depth 128.
  C4  SoC-shaped, ~10M ANDs, 256K flops, 24 RAM blocks (8 tiles + uncore).
  C5  = C3 netlist (streams differ, see gen/stimulus.py).

Nothing here evaluates the circuit; the module only draws structure with
numpy's PCG64 and writes `.eaig` files (gen/aig.py).
"""
from __future__ import annotations

import dataclasses
import os
from typing import Dict, List, Optional

import numpy as np

from .aig import AigBuilder, Netlist, RamBlock, write_eaig, RAM_ABITS, RAM_DBITS


# ==========================================================================
# C1: counter + adder + LFSR
# ==========================================================================

C1_LFSR_RESET = 0xACE1
C1_LFSR_TAPS = (15, 13, 12, 10)   # x^16 + x^14 + x^13 + x^11 + 1 (Fibonacci)


def build_c1() -> Netlist:
    """PIs (35): rst, en, cin, a[32].  Flops (64): cnt[32], lfsr[16], r[16].

    cnt'  = rst ? 0 : cnt + en
    lfsr' = rst ? 0xACE1 : ((lfsr << 1) & 0xFFFF) | (l15 ^ l13 ^ l12 ^ l10)
    r'    = rst ? 0 : s[15:0] ^ lfsr
    s, cout = cnt + a + cin            (32-bit ripple carry)
    POs (97): s[32], cout, cnt[32], lfsr[16], r[16]
    """
    b = AigBuilder("c1")
    rst, en, cin = b.input(), b.input(), b.input()
    a = b.inputs_n(32)
    cnt = [b.latch() for _ in range(32)]
    lfsr = [b.latch() for _ in range(16)]
    r = [b.latch() for _ in range(16)]
    nrst = b.NOT(rst)
    # counter: half-adder incrementer
    carry = en
    for i in range(32):
        s_i = b.XOR(cnt[i], carry)
        carry = b.AND(cnt[i], carry)
        b.set_next(cnt[i], b.AND(nrst, s_i))
    # lfsr
    fb = b.XOR(b.XOR(lfsr[15], lfsr[13]), b.XOR(lfsr[12], lfsr[10]))
    shifted = [fb] + lfsr[:15]
    for i in range(16):
        if (C1_LFSR_RESET >> i) & 1:
            b.set_next(lfsr[i], b.OR(rst, shifted[i]))
        else:
            b.set_next(lfsr[i], b.AND(nrst, shifted[i]))
    # adder
    s = []
    c = cin
    for i in range(32):
        si, c = b.full_adder(cnt[i], a[i], c)
        s.append(si)
    cout = c
    for i in range(16):
        b.set_next(r[i], b.AND(nrst, b.XOR(s[i], lfsr[i])))
    for x in s:
        b.output(x)
    b.output(cout)
    for x in cnt + lfsr + r:
        b.output(x)
    return b.finish()


# ==========================================================================
# G family: cluster-structured, levelised, long-tailed AIG
# ==========================================================================

@dataclasses.dataclass
class ClusterSpec:
    n_and: int          # target ANDs before pruning (calibrated)
    n_flop: int
    d_max: int          # deepest level of this cluster
    tau: float          # width profile decay w(l) ~ exp(-(l-1)/tau)
    n_tail: int = 0     # number of carry-chain tails (0 = none)
    d_head: int = 0     # head depth (0 = auto: where the profile reaches ~1 node)
    group: int = 0      # cross-cluster picks stay inside a group


@dataclasses.dataclass
class RamMacroSpec:
    owner: int              # cluster that computes the write ports
    readers: List[int]      # clusters whose level-0 sources include rdata
    n_blocks: int = 1       # 1 or 4 (4 = 15-bit address with decode adapter)


@dataclasses.dataclass
class GSpec:
    name: str
    clusters: List[ClusterSpec]
    n_pi: int
    n_po: int
    p_x: float
    rams: List[RamMacroSpec] = dataclasses.field(default_factory=list)
    reset_pi0: bool = False     # PI0 = sync reset ANDed into every flop D
    pi_per_cluster: int = 16
    neighbour_flops: int = 64   # flop Q's of each neighbouring cluster used as sources


def _geom0(rng, p, n):
    return rng.geometric(p, size=n) - 1


def build_G(spec: GSpec, seed: int, scale: float = 1.0) -> (Netlist, dict):
    rng = np.random.Generator(np.random.PCG64(seed))
    C = len(spec.clusters)
    # ---- inputs: PIs then RAM rdata inputs --------------------------------
    n_blocks = sum(m.n_blocks for m in spec.rams)
    n_inputs = spec.n_pi + RAM_DBITS * n_blocks
    n_flop_total = sum(c.n_flop for c in spec.clusters)
    n_adapter_flops = sum(2 for m in spec.rams if m.n_blocks == 4)
    L = n_flop_total + n_adapter_flops
    I = n_inputs
    var_pi = 1 + np.arange(spec.n_pi, dtype=np.int64)
    var_rdata = 1 + spec.n_pi + np.arange(RAM_DBITS * n_blocks, dtype=np.int64)
    flop_base = np.zeros(C + 1, dtype=np.int64)
    np.cumsum([c.n_flop for c in spec.clusters], out=flop_base[1:])
    var_flop = 1 + I + np.arange(L, dtype=np.int64)   # includes adapter flops at the end
    next_var = 1 + I + L

    # AND storage (lits in final numbering); filled in blocks
    rhs0_blocks: List[np.ndarray] = []
    rhs1_blocks: List[np.ndarray] = []
    lvl_blocks: List[np.ndarray] = []

    def add_ands(a: np.ndarray, b: np.ndarray, lvl: np.ndarray) -> np.ndarray:
        nonlocal next_var
        n = len(a)
        ids = next_var + np.arange(n, dtype=np.int64)
        next_var += n
        rhs0_blocks.append(a.astype(np.int64))
        rhs1_blocks.append(b.astype(np.int64))
        lvl_blocks.append(lvl.astype(np.int32))
        return ids

    # ---- RAM macro adapters on the read side (level-0-ish sources) ---------
    # For 4-block macros the read data is muxed by a registered copy of the two
    # high address bits (adapter logic); built after the flops exist.
    blk = 0
    macro_rdata_lits: List[np.ndarray] = []   # 32 lits per macro fed to readers
    macro_blocks: List[List[int]] = []
    adapter_flop_idx = n_flop_total
    adapter_flops: List[tuple] = []           # (flop index, macro idx, bit)
    for mi, m in enumerate(spec.rams):
        blocks = list(range(blk, blk + m.n_blocks))
        blk += m.n_blocks
        macro_blocks.append(blocks)
        if m.n_blocks == 1:
            macro_rdata_lits.append(2 * var_rdata[blocks[0] * 32:(blocks[0] + 1) * 32])
        else:
            assert m.n_blocks == 4
            s0 = 2 * var_flop[adapter_flop_idx]
            s1 = 2 * var_flop[adapter_flop_idx + 1]
            adapter_flops.append((adapter_flop_idx, mi, 0))
            adapter_flops.append((adapter_flop_idx + 1, mi, 1))
            adapter_flop_idx += 2
            dec = []
            for bsel in range(4):
                x0 = s0 ^ (0 if bsel & 1 else 1)
                x1 = s1 ^ (0 if bsel & 2 else 1)
                dec.append(add_ands(np.array([x0]), np.array([x1]), np.array([1]))[0] * 2)
            terms = []
            for bsel, bb in enumerate(blocks):
                rd = 2 * var_rdata[bb * 32:(bb + 1) * 32]
                terms.append(2 * add_ands(rd, np.full(32, dec[bsel]), np.full(32, 2)))
            o01 = 2 * add_ands(terms[0] ^ 1, terms[1] ^ 1, np.full(32, 3)) ^ 1
            o23 = 2 * add_ands(terms[2] ^ 1, terms[3] ^ 1, np.full(32, 3)) ^ 1
            mux = 2 * add_ands(o01 ^ 1, o23 ^ 1, np.full(32, 4)) ^ 1
            macro_rdata_lits.append(mux)

    # ---- level-0 sources per cluster --------------------------------------
    sources: List[np.ndarray] = []
    for c, cs in enumerate(spec.clusters):
        src = [2 * var_flop[flop_base[c]:flop_base[c + 1]]]
        for nb in (c - 1, c + 1):
            nb %= C
            if nb != c:
                lo, hi = flop_base[nb], flop_base[nb + 1]
                k = min(spec.neighbour_flops, hi - lo)
                src.append(2 * var_flop[lo + rng.choice(hi - lo, size=k, replace=False)])
        k = min(spec.pi_per_cluster, spec.n_pi - (1 if spec.reset_pi0 else 0))
        pis = rng.choice(np.arange(1 if spec.reset_pi0 else 0, spec.n_pi), size=k, replace=False)
        src.append(2 * var_pi[pis])
        for mi, m in enumerate(spec.rams):
            if c in m.readers:
                src.append(macro_rdata_lits[mi])
        sources.append(np.concatenate(src).astype(np.int64))
    src_off = np.zeros(C + 1, dtype=np.int64)
    np.cumsum([len(s) for s in sources], out=src_off[1:])
    src_all = np.concatenate(sources)

    # ---- widths per (cluster, level) -------------------------------------
    Dg = max(c.d_max for c in spec.clusters)
    W = np.zeros((C, Dg + 1), dtype=np.int64)
    head = np.zeros(C, dtype=np.int64)
    for c, cs in enumerate(spec.clusters):
        n_tail_nodes = 0
        if cs.n_tail:
            dh = cs.d_head if cs.d_head else max(8, int(round(cs.tau * 6)))
            dh = min(dh, cs.d_max)
            n_tail_nodes = cs.n_tail * (cs.d_max - dh)
        else:
            dh = cs.d_max
        n_head = max(dh, int(cs.n_and * scale) - n_tail_nodes)
        ls = np.arange(1, dh + 1)
        prof = np.exp(-(ls - 1) / cs.tau)
        w = np.maximum(1, np.round(n_head * prof / prof.sum())).astype(np.int64)
        W[c, 1:dh + 1] = w
        if cs.n_tail:
            W[c, dh + 1:cs.d_max + 1] = cs.n_tail
        head[c] = dh
    top = np.array([c.d_max for c in spec.clusters], dtype=np.int64)
    groups = np.array([c.group for c in spec.clusters], dtype=np.int64)
    # groups are contiguous cluster ranges
    gstart = np.zeros(groups.max() + 1, dtype=np.int64)
    gsize = np.zeros(groups.max() + 1, dtype=np.int64)
    for g in np.unique(groups):
        mem = np.where(groups == g)[0]
        assert np.all(np.diff(mem) == 1), "cluster groups must be contiguous"
        gstart[g], gsize[g] = mem[0], len(mem)

    # start id of (cluster, level) block
    start = np.zeros((C, Dg + 1), dtype=np.int64)
    for l in range(1, Dg + 1):
        n_l = int(W[:, l].sum())
        if n_l == 0:
            continue
        cl = np.repeat(np.arange(C), W[:, l])
        # input 0: level l-1, same cluster (pins the exact level)
        if l == 1:
            u = rng.random(n_l)
            ln = (src_off[cl + 1] - src_off[cl])
            in0 = src_all[src_off[cl] + (u * ln).astype(np.int64)]
        else:
            is_tail = l > head[cl]
            u = rng.random(n_l)
            idx = (u * W[cl, l - 1]).astype(np.int64)
            # tail chains: node k continues chain k of level l-1
            pos_in_level = np.arange(n_l) - np.repeat(np.cumsum(W[:, l]) - W[:, l], W[:, l])
            idx = np.where(is_tail & (W[cl, l - 1] == W[cl, l]), pos_in_level, idx)
            in0 = 2 * (start[cl, l - 1] + idx)
        # input 1: level drawn geometrically toward l-1, maybe another cluster
        g = _geom0(rng, 0.45, n_l)
        l1 = np.maximum(0, l - 1 - g)
        is_tail = l > head[cl]
        l1 = np.where(is_tail, rng.integers(0, np.minimum(7, l), size=n_l), l1)
        cross = rng.random(n_l) < spec.p_x
        gs = gstart[groups[cl]]
        gz = gsize[groups[cl]]
        hop = 1 + (rng.random(n_l) * np.maximum(gz - 1, 1)).astype(np.int64)
        c1 = np.where(cross & (gz > 1), gs + (cl - gs + hop) % np.maximum(gz, 1), cl)
        l1 = np.minimum(l1, top[c1])
        # cross-cluster fan-ins come from shallow levels of the other cluster
        # (module-interface logic), so cones leak across clusters only a little
        l1 = np.where(c1 != cl, np.minimum(rng.integers(0, 4, size=n_l), l - 1), l1)
        in1 = np.empty(n_l, dtype=np.int64)
        z = l1 == 0
        if np.any(z):
            u = rng.random(int(z.sum()))
            ln = src_off[c1[z] + 1] - src_off[c1[z]]
            in1[z] = src_all[src_off[c1[z]] + (u * ln).astype(np.int64)]
        nz = ~z
        if np.any(nz):
            u = rng.random(int(nz.sum()))
            in1[nz] = 2 * (start[c1[nz], l1[nz]] + (u * W[c1[nz], l1[nz]]).astype(np.int64))
        neg = rng.integers(0, 2, size=(2, n_l))
        ids = add_ands(in0 ^ neg[0], in1 ^ neg[1], np.full(n_l, l))
        # record block starts per cluster at this level
        cs_ = np.cumsum(W[:, l]) - W[:, l]
        start[:, l] = ids[0] + cs_

    def pick_nodes(c: int, n: int, deep_frac: float) -> np.ndarray:
        """n literals from cluster c: deep_frac from the deepest third of levels."""
        t = top[c]
        nd = int(round(n * deep_frac))
        lv_lo = max(1, int(np.ceil(2 * t / 3)))
        deep_levels = np.arange(lv_lo, t + 1)
        all_levels = np.arange(1, t + 1)
        out = []
        for levels, k in ((deep_levels, nd), (all_levels, n - nd)):
            if k == 0:
                continue
            wts = W[c, levels].astype(np.float64)
            cum = np.cumsum(wts)
            r = rng.random(k) * cum[-1]
            li = np.searchsorted(cum, r, side="right")
            li = np.minimum(li, len(levels) - 1)
            lv = levels[li]
            off = (rng.random(k) * W[c, lv]).astype(np.int64)
            out.append(2 * (start[c, lv] + off))
        lits = np.concatenate(out) if out else np.zeros(0, dtype=np.int64)
        return lits ^ rng.integers(0, 2, size=len(lits))

    # ---- flop D endpoints -------------------------------------------------
    latch_next = np.zeros(L, dtype=np.int64)
    for c, cs in enumerate(spec.clusters):
        d = pick_nodes(c, cs.n_flop, 0.5)
        latch_next[flop_base[c]:flop_base[c + 1]] = rng.permutation(d)
    # ---- RAM write ports ----------------------------------------------------
    rams: List[RamBlock] = []
    for mi, m in enumerate(spec.rams):
        oc = m.owner
        fl = 2 * var_flop[flop_base[oc]:flop_base[oc + 1]]
        abits = RAM_ABITS + (2 if m.n_blocks == 4 else 0)
        sel = rng.choice(len(fl), size=abits + 3, replace=False)
        raddr = fl[sel[:abits]]
        waddr = raddr.copy()
        waddr[:3] = fl[sel[abits:abits + 3]]   # high bits shared -> frequent same-address R/W (U8)
        wdata = pick_nodes(oc, RAM_DBITS, 0.3)
        wbe = pick_nodes(oc, RAM_DBITS, 0.3)
        if m.n_blocks == 1:
            bb = macro_blocks[mi][0]
            rams.append(RamBlock(rdata=list(range(spec.n_pi + 32 * bb, spec.n_pi + 32 * (bb + 1))),
                                 raddr=[int(x) for x in raddr], waddr=[int(x) for x in waddr],
                                 wdata=[int(x) for x in wdata], wbe=[int(x) for x in wbe]))
        else:
            wa_hi = waddr[13:15]
            dec = []
            for bsel in range(4):
                x0 = wa_hi[0] ^ (0 if bsel & 1 else 1)
                x1 = wa_hi[1] ^ (0 if bsel & 2 else 1)
                dec.append(2 * add_ands(np.array([x0]), np.array([x1]), np.array([Dg + 1]))[0])
            for bsel, bb in enumerate(macro_blocks[mi]):
                wbe_b = 2 * add_ands(wbe, np.full(32, dec[bsel]), np.full(32, Dg + 2))
                rams.append(RamBlock(rdata=list(range(spec.n_pi + 32 * bb, spec.n_pi + 32 * (bb + 1))),
                                     raddr=[int(x) for x in raddr[:13]], waddr=[int(x) for x in waddr[:13]],
                                     wdata=[int(x) for x in wdata], wbe=[int(x) for x in wbe_b]))
            for fidx, mj, bit in adapter_flops:
                if mj == mi:
                    latch_next[fidx] = raddr[13 + bit]
    # ---- sync reset -------------------------------------------------------
    if spec.reset_pi0:
        nrst = 2 * var_pi[0] ^ 1
        ids = add_ands(np.full(n_flop_total, nrst), latch_next[:n_flop_total], np.full(n_flop_total, Dg + 3))
        latch_next[:n_flop_total] = 2 * ids
    # ---- POs ---------------------------------------------------------------
    po_cl = rng.integers(0, C, size=spec.n_po)
    outputs = np.zeros(spec.n_po, dtype=np.int64)
    for c in np.unique(po_cl):
        k = np.where(po_cl == c)[0]
        outputs[k] = pick_nodes(int(c), len(k), 1.0)

    rhs0 = np.concatenate(rhs0_blocks)
    rhs1 = np.concatenate(rhs1_blocks)
    A = len(rhs0)
    # true logic level of every AND (blocks have no internal dependencies)
    base = 1 + I + L
    lev = np.zeros(A, dtype=np.int32)
    off = 0
    for b0, b1 in zip(rhs0_blocks, rhs1_blocks):
        n = len(b0)
        v0 = (b0 >> 1) - base
        v1 = (b1 >> 1) - base
        l0 = np.where(v0 >= 0, lev[np.maximum(v0, 0)], 0)
        l1_ = np.where(v1 >= 0, lev[np.maximum(v1, 0)], 0)
        lev[off:off + n] = 1 + np.maximum(l0, l1_)
        off += n
    net = _prune(I, L, latch_next, outputs, rhs0, rhs1, rams, spec.name, lev)
    return net, dict(generated_ands=A)


def _prune(I, L, latch_next, outputs, rhs0, rhs1, rams, name, lev) -> Netlist:
    """Cone-of-influence pruning from all endpoints, keeping topological order."""
    A = len(rhs0)
    base = 1 + I + L
    live = np.zeros(A, dtype=bool)
    roots = [latch_next, outputs]
    for r in rams:
        roots += [np.array(r.raddr), np.array(r.waddr), np.array(r.wdata), np.array(r.wbe)]
    rv = np.concatenate([np.asarray(x, dtype=np.int64) for x in roots]) >> 1
    rv = rv[rv >= base] - base
    live[rv] = True
    v0 = (rhs0 >> 1) - base
    v1 = (rhs1 >> 1) - base
    order = np.argsort(-lev, kind="stable")
    bounds = np.searchsorted(-lev[order], np.arange(-int(lev.max()), 0), side="left")
    bounds = np.append(bounds, A)
    for k in range(len(bounds) - 1):
        sel = order[bounds[k]:bounds[k + 1]]
        sel = sel[live[sel]]
        a = v0[sel]; b = v1[sel]
        live[a[a >= 0]] = True
        live[b[b >= 0]] = True
    keep = np.where(live)[0]
    newid = np.full(A, -1, dtype=np.int64)
    newid[keep] = np.arange(len(keep))

    def remap(lits):
        lits = np.asarray(lits, dtype=np.int64)
        v = lits >> 1
        out = lits.copy()
        m = v >= base
        nv = newid[v[m] - base]
        assert np.all(nv >= 0)
        out[m] = 2 * (base + nv) + (lits[m] & 1)
        return out

    n_rhs0 = remap(rhs0[keep])
    n_rhs1 = remap(rhs1[keep])
    rams2 = [RamBlock(rdata=r.rdata, raddr=remap(r.raddr).tolist(), waddr=remap(r.waddr).tolist(),
                      wdata=remap(r.wdata).tolist(), wbe=remap(r.wbe).tolist()) for r in rams]
    return Netlist(n_inputs=I, latch_next=remap(latch_next).astype(np.uint64),
                   latch_init=np.zeros(L, dtype=np.uint8), outputs=remap(outputs).astype(np.uint64),
                   and_rhs0=n_rhs0.astype(np.uint64), and_rhs1=n_rhs1.astype(np.uint64),
                   rams=rams2, name=name)


# ==========================================================================
# config specs
# ==========================================================================

def spec_c2() -> GSpec:
    K = 16
    cl = [ClusterSpec(n_and=100_000 // K, n_flop=4096 // K, d_max=40, tau=6.0) for _ in range(K)]
    return GSpec("c2", cl, n_pi=128, n_po=128, p_x=0.02)


def _c3_clusters(K=64, n_and=1_000_000, n_flop=32768, d_max=128, group=0, tail_every=4):
    cl = []
    for c in range(K):
        tail = 32 if (c % tail_every) == 0 else 0
        cl.append(ClusterSpec(n_and=n_and // K, n_flop=n_flop // K,
                              d_max=d_max if tail else 48, tau=6.0, n_tail=tail,
                              d_head=48 if tail else 0, group=group))
    return cl


def spec_c3() -> GSpec:
    cl = _c3_clusters()
    rams = [RamMacroSpec(owner=3, readers=[3, 10, 20, 30]),
            RamMacroSpec(owner=40, readers=[40, 45, 50, 60])]
    return GSpec("c3", cl, n_pi=256, n_po=256, p_x=0.01, rams=rams, reset_pi0=True)


def spec_c4() -> GSpec:
    cl: List[ClusterSpec] = []
    rams: List[RamMacroSpec] = []
    K = 64
    for t in range(8):
        base = len(cl)
        cl += _c3_clusters(K=K, n_and=1_100_000, n_flop=28_672, d_max=150, group=t)
        rams.append(RamMacroSpec(owner=base + 3, readers=[base + 3, base + 10, base + 20, base + 30]))
        rams.append(RamMacroSpec(owner=base + 40, readers=[base + 40, base + 45, base + 50, base + 60]))
    base = len(cl)
    cl += _c3_clusters(K=K, n_and=1_200_000, n_flop=32_768, d_max=150, group=8)
    rams.append(RamMacroSpec(owner=base + 5, readers=[base + 5, base + 15, base + 25, base + 35], n_blocks=4))
    rams.append(RamMacroSpec(owner=base + 50, readers=[base + 50, base + 55, base + 60, base + 2], n_blocks=4))
    return GSpec("c4", cl, n_pi=512, n_po=512, p_x=0.01, rams=rams, reset_pi0=True)


SPECS = {"c2": (spec_c2, 2, 100_000), "c3": (spec_c3, 3, 1_000_000), "c4": (spec_c4, 4, 10_000_000)}


def build_config(cfg: str) -> Netlist:
    """Deterministic netlist for a config name ('c1'..'c5'); C5 reuses C3."""
    cfg = cfg.lower()
    if cfg == "c1":
        return build_c1()
    if cfg == "c5":
        cfg = "c3"
    fn, seed, target = SPECS[cfg]
    spec = fn()
    # two-pass calibration so that the *live* AND count lands near the target
    scale = 1.0
    for _ in range(3):
        net, info = build_G(spec, seed, scale=scale)
        ratio = net.n_ands / target
        if abs(ratio - 1) <= 0.02:
            break
        scale /= ratio
    net.name = cfg
    return net


def netlist_path(cfg: str, cache_dir: Optional[str] = None) -> str:
    """Generate (once) and cache the `.eaig` for a config; returns the path."""
    cfg = cfg.lower()
    if cfg == "c5":
        cfg = "c3"
    cache_dir = cache_dir or os.environ.get("GEM_CACHE", os.path.join(os.path.dirname(os.path.dirname(
        os.path.abspath(__file__))), ".cache"))
    os.makedirs(cache_dir, exist_ok=True)
    p = os.path.join(cache_dir, f"{cfg}.eaig")
    if not os.path.exists(p):
        net = build_config(cfg)
        tmp = p + f".tmp{os.getpid()}"
        write_eaig(net, tmp)
        os.replace(tmp, p)
    return p
