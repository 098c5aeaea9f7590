"""Python twin of the oracle -- TEST INFRASTRUCTURE ONLY.

A deliberately *different* evaluator of the same plain definition
(SURVEY §8(c)): it parses the `.eaig` itself and evaluates every endpoint by
memoised recursion over the DAG (no topological sort, no levelisation).  Used
to cross-check oracle.cpp on small circuits and short prefixes.

Semantics (U5-U12):
per cycle t: apply PI[t]; RAM rdata inputs read the registered read data; POs
are sampled before the edge; latches take next; each RAM reads M[raddr]
before writing M[waddr] = (M & ~wbe) | (wdata & wbe).
"""
from __future__ import annotations

import sys
from typing import Dict, List

import numpy as np


def _varint(buf: bytes, pos: int):
    x = 0
    shift = 0
    while True:
        b = buf[pos]
        pos += 1
        x |= (b & 0x7F) << shift
        if not b & 0x80:
            return x, pos
        shift += 7


class Twin:
    def __init__(self, path: str):
        data = open(path, "rb").read()
        nl = data.index(b"\n")
        hdr = data[:nl].split()
        fmt = hdr[0].decode()
        M, I, L, O, A = (int(x) for x in hdr[1:6])
        self.I, self.L, self.O, self.A = I, L, O, A
        pos = nl + 1
        lines = []

        def next_line():
            nonlocal pos
            e = data.index(b"\n", pos)
            s = data[pos:e].decode()
            pos = e + 1
            return s

        if fmt == "aag":
            for i in range(I):
                assert int(next_line()) == 2 * (i + 1)
        self.latch_next = []
        self.latch_init = []
        for j in range(L):
            f = next_line().split()
            if fmt == "aag":
                f = f[1:]
            self.latch_next.append(int(f[0]))
            cur = 2 * (I + 1 + j)
            init = int(f[1]) if len(f) > 1 else 0
            self.latch_init.append(1 if init == 1 else 0)
        self.outputs = [int(next_line()) for _ in range(O)]
        self.ands: Dict[int, tuple] = {}
        if fmt == "aag":
            for _ in range(A):
                a, b, c = (int(x) for x in next_line().split())
                self.ands[a >> 1] = (b, c)
        else:
            for k in range(A):
                lhs = 2 * (I + L + 1 + k)
                d0, pos = _varint(data, pos)
                d1, pos = _varint(data, pos)
                r0 = lhs - d0
                self.ands[lhs >> 1] = (r0, r0 - d1)
        self.rams = []
        rest = data[pos:].decode(errors="replace").splitlines()
        in_c = False
        for ln in rest:
            if not in_c:
                if ln == "c" or ln.startswith("c "):
                    in_c = True
                continue
            if ln.startswith("gem-ram "):
                f = dict(kv.split("=") for kv in ln.split()[2:])
                g = lambda k: [int(x) for x in f[k].split(",")]
                self.rams.append(dict(rdata=g("rdata"), raddr=g("raddr"), waddr=g("waddr"),
                                      wdata=g("wdata"), wbe=g("wbe")))
        ram_in = {}
        for r, ram in enumerate(self.rams):
            for k, inp in enumerate(ram["rdata"]):
                ram_in[inp] = (r, k)
        self.ram_in = ram_in
        self.pi_of_input = {}
        p = 0
        for i in range(I):
            if i not in ram_in:
                self.pi_of_input[i] = p
                p += 1
        self.n_pi = p
        self.reset()

    def reset(self):
        self.Q = list(self.latch_init)
        self.RD = [0] * len(self.rams)
        self.MEM = [dict() for _ in self.rams]

    def run(self, stim_bits: np.ndarray):
        """stim_bits uint8[cycles][n_pi] -> (po_bits[cycles][O], q_bits[cycles][L])."""
        sys.setrecursionlimit(max(10000, 4 * self.A + 100))
        po_tr, q_tr = [], []
        I = self.I
        for t in range(stim_bits.shape[0]):
            memo = {}

            def var(v):
                if v == 0:
                    return 0
                if v <= I:
                    i = v - 1
                    if i in self.ram_in:
                        r, k = self.ram_in[i]
                        return (self.RD[r] >> k) & 1
                    return int(stim_bits[t, self.pi_of_input[i]])
                if v <= I + self.L:
                    return self.Q[v - I - 1]
                if v in memo:
                    return memo[v]
                a, b = self.ands[v]
                r = lit(a) & lit(b)
                memo[v] = r
                return r

            def lit(l):
                return var(l >> 1) ^ (l & 1)

            po_tr.append([lit(o) for o in self.outputs])
            qn = [lit(x) for x in self.latch_next]
            rdn = []
            for r, ram in enumerate(self.rams):
                num = lambda ls: sum(lit(x) << k for k, x in enumerate(ls))
                ra, wa, wd, be = num(ram["raddr"]), num(ram["waddr"]), num(ram["wdata"]), num(ram["wbe"])
                mem = self.MEM[r]
                rdn.append(mem.get(ra, 0))
                mem[wa] = (mem.get(wa, 0) & ~be & 0xFFFFFFFF) | (wd & be)
            self.Q = qn
            self.RD = rdn
            q_tr.append(list(self.Q))
        n = len(po_tr)
        return np.array(po_tr, np.uint8).reshape(n, self.O), np.array(q_tr, np.uint8).reshape(n, self.L)
