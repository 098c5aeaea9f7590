"""E-AIG netlist container, builder and `.eaig` writer (shared INPUT side).

This module is part of the seeded *input generators* (``gen/``).  It builds
and serialises synchronous extended AIGs; it holds none of the simulation
arithmetic, so both the CPU oracle (``oracle/``) and the CUDA path
(mapper + libgem) consume its files without sharing any evaluation code.

E-AIG (§III-A): 2-input ANDs with inverted edges, D flip-flops
and native RAM blocks of 13-bit address x 32-bit data (§III-B).

File format ``.eaig`` (SURVEY.md §8(c) "Netlist model"):
  * AIGER 1.9, ASCII ``aag`` or binary ``aig``, header ``M I L O A``
    (B/C/J/F sections are not allowed).
  * literal = 2*var + neg, var 0 = constant FALSE.
  * latch ``cur next [init]`` with init in {0, 1, cur}; ``cur`` (uninitialised)
    is read as 0 (reading U5).
  * RAM blocks live in the comment section, one line per block::

        gem-ram <id> rdata=<32 input indices> raddr=<13 lits> waddr=<13 lits> wdata=<32 lits> wbe=<32 lits>

    The 32 ``rdata`` signals are AIGER *inputs* driven by the RAM; they are
    removed from the primary-input numbering used for stimulus.
"""
from __future__ import annotations

import dataclasses
from typing import List, Optional, Sequence

import numpy as np

RAM_ABITS = 13   # P:93 "13 bits address"
RAM_DBITS = 32   # P:93 "32 bits data"


@dataclasses.dataclass
class RamBlock:
    rdata: List[int]        # 32 AIGER input indices (0-based) driven by the RAM
    raddr: List[int]        # 13 literals
    waddr: List[int]        # 13 literals
    wdata: List[int]        # 32 literals
    wbe: List[int]          # 32 literals (per-bit write enable, reading U9)


@dataclasses.dataclass
class Netlist:
    """AIGER-numbered netlist.

    vars 1..I are inputs, I+1..I+L latches, I+L+1..I+L+A ANDs (topological).
    """
    n_inputs: int
    latch_next: np.ndarray          # uint64 literals, len L
    latch_init: np.ndarray          # uint8: 0, 1 or 2 (= uninitialised, reads 0)
    outputs: np.ndarray             # uint64 literals, len O
    and_rhs0: np.ndarray            # uint64 literals, len A
    and_rhs1: np.ndarray            # uint64 literals, len A
    rams: List[RamBlock] = dataclasses.field(default_factory=list)
    name: str = ""

    @property
    def n_latches(self) -> int:
        return int(len(self.latch_next))

    @property
    def n_outputs(self) -> int:
        return int(len(self.outputs))

    @property
    def n_ands(self) -> int:
        return int(len(self.and_rhs0))

    @property
    def max_var(self) -> int:
        return self.n_inputs + self.n_latches + self.n_ands

    def ram_input_set(self) -> set:
        s = set()
        for r in self.rams:
            s.update(r.rdata)
        return s

    @property
    def n_pi(self) -> int:
        """Primary inputs = AIGER inputs minus RAM rdata inputs."""
        return self.n_inputs - len(self.ram_input_set())

    def pi_input_indices(self) -> np.ndarray:
        """AIGER input index of each primary input, in PI order."""
        ram = self.ram_input_set()
        return np.array([i for i in range(self.n_inputs) if i not in ram], dtype=np.int64)

    def stats(self) -> dict:
        return dict(name=self.name, n_inputs=self.n_inputs, n_pi=self.n_pi,
                    n_latches=self.n_latches, n_outputs=self.n_outputs,
                    n_ands=self.n_ands, n_rams=len(self.rams))


# --------------------------------------------------------------------------
# writer
# --------------------------------------------------------------------------

def _ram_lines(net: Netlist) -> List[str]:
    out = []
    for k, r in enumerate(net.rams):
        assert len(r.rdata) == RAM_DBITS and len(r.raddr) == RAM_ABITS
        assert len(r.waddr) == RAM_ABITS and len(r.wdata) == RAM_DBITS and len(r.wbe) == RAM_DBITS
        j = lambda xs: ",".join(str(int(x)) for x in xs)
        out.append(f"gem-ram {k} rdata={j(r.rdata)} raddr={j(r.raddr)} "
                   f"waddr={j(r.waddr)} wdata={j(r.wdata)} wbe={j(r.wbe)}")
    return out


def _varint_bytes(vals: np.ndarray) -> bytes:
    """AIGER binary delta encoding (7-bit little-endian groups), vectorised."""
    vals = vals.astype(np.uint64)
    n = len(vals)
    if n == 0:
        return b""
    nbytes = np.ones(n, dtype=np.int64)
    v = vals >> np.uint64(7)
    while np.any(v):
        nbytes += (v != 0)
        v = v >> np.uint64(7)
    total = int(nbytes.sum())
    out = np.zeros(total, dtype=np.uint8)
    starts = np.zeros(n, dtype=np.int64)
    np.cumsum(nbytes[:-1], out=starts[1:])
    v = vals.copy()
    for k in range(int(nbytes.max())):
        active = nbytes > k
        idx = starts[active] + k
        byte = (v[active] & np.uint64(0x7F)).astype(np.uint8)
        more = nbytes[active] > k + 1
        byte = byte | (more.astype(np.uint8) << 7)
        out[idx] = byte
        v = v >> np.uint64(7)
    return out.tobytes()


def write_eaig(net: Netlist, path: str, binary: Optional[bool] = None) -> None:
    I, L, O, A = net.n_inputs, net.n_latches, net.n_outputs, net.n_ands
    M = I + L + A
    if binary is None:
        binary = A > 200_000
    lat_init = net.latch_init
    lines_latch = []
    for j in range(L):
        init = int(lat_init[j])
        cur = 2 * (I + 1 + j)
        nxt = int(net.latch_next[j])
        if init == 0:
            tail = ""
        elif init == 1:
            tail = " 1"
        else:
            tail = f" {cur}"
        lines_latch.append((cur, nxt, tail))
    with open(path, "wb") as f:
        if not binary:
            hdr = f"aag {M} {I} {L} {O} {A}\n"
            f.write(hdr.encode())
            f.write("".join(f"{2 * (i + 1)}\n" for i in range(I)).encode())
            f.write("".join(f"{c} {n}{t}\n" for c, n, t in lines_latch).encode())
            f.write("".join(f"{int(o)}\n" for o in net.outputs).encode())
            lhs = 2 * (I + L + 1 + np.arange(A, dtype=np.int64))
            body = np.stack([lhs, net.and_rhs0.astype(np.int64), net.and_rhs1.astype(np.int64)], 1)
            chunk = 1 << 18
            for s in range(0, A, chunk):
                b = body[s:s + chunk]
                f.write(("\n".join(f"{x} {y} {z}" for x, y, z in b.tolist()) + ("\n" if len(b) else "")).encode())
        else:
            hdr = f"aig {M} {I} {L} {O} {A}\n"
            f.write(hdr.encode())
            f.write("".join(f"{n}{t}\n" for c, n, t in lines_latch).encode())
            f.write("".join(f"{int(o)}\n" for o in net.outputs).encode())
            lhs = 2 * (I + L + 1 + np.arange(A, dtype=np.uint64))
            r0 = net.and_rhs0.astype(np.uint64)
            r1 = net.and_rhs1.astype(np.uint64)
            hi = np.maximum(r0, r1)
            lo = np.minimum(r0, r1)
            assert np.all(hi < lhs), "ANDs must be topologically ordered"
            d0 = lhs - hi
            d1 = hi - lo
            inter = np.empty(2 * A, dtype=np.uint64)
            inter[0::2] = d0
            inter[1::2] = d1
            f.write(_varint_bytes(inter))
        f.write(b"c\n")
        f.write(("\n".join(_ram_lines(net)) + "\n").encode() if net.rams else b"")
        if net.name:
            f.write(f"gem-name {net.name}\n".encode())


# --------------------------------------------------------------------------
# small builder (C1 and test circuits)
# --------------------------------------------------------------------------

class AigBuilder:
    """Tiny structural builder; no simplification (structure is kept as built).

    Internal node ids are assigned in creation order; `finish()` renumbers to
    AIGER order (inputs, latches, ANDs).  Literals handed out by the builder
    are internal literals (2*id + neg); id 0 is constant FALSE.
    """
    FALSE = 0
    TRUE = 1

    def __init__(self, name: str = ""):
        self.name = name
        self.kind = [("c", 0)]      # id -> (kind, index)
        self.inputs: List[int] = []
        self.latches: List[int] = []
        self.latch_next: List[Optional[int]] = []
        self.latch_init: List[int] = []
        self.ands: List[tuple] = []   # (id, a, b)
        self.outputs: List[int] = []
        self.rams: List[dict] = []

    def _new(self, kind):
        self.kind.append(kind)
        return len(self.kind) - 1

    def input(self) -> int:
        i = self._new(("i", len(self.inputs)))
        self.inputs.append(i)
        return 2 * i

    def inputs_n(self, n: int) -> List[int]:
        return [self.input() for _ in range(n)]

    def latch(self, init: int = 0) -> int:
        i = self._new(("l", len(self.latches)))
        self.latches.append(i)
        self.latch_next.append(None)
        self.latch_init.append(init)
        return 2 * i

    def set_next(self, latch_lit: int, nxt: int) -> None:
        idx = self.kind[latch_lit >> 1][1]
        self.latch_next[idx] = nxt

    def AND(self, a: int, b: int) -> int:
        i = self._new(("a", len(self.ands)))
        self.ands.append((i, a, b))
        return 2 * i

    @staticmethod
    def NOT(a: int) -> int:
        return a ^ 1

    def OR(self, a, b):
        return self.AND(a ^ 1, b ^ 1) ^ 1

    def XOR(self, a, b):
        # 3 ANDs: (a | b) & !(a & b)
        return self.AND(self.OR(a, b), self.AND(a, b) ^ 1)

    def MUX(self, s, a, b):
        """s ? a : b"""
        return self.OR(self.AND(s, a), self.AND(s ^ 1, b))

    def MAJ(self, a, b, c):
        return self.OR(self.OR(self.AND(a, b), self.AND(a, c)), self.AND(b, c))

    def full_adder(self, a, b, c):
        s = self.XOR(self.XOR(a, b), c)
        co = self.MAJ(a, b, c)
        return s, co

    def output(self, lit: int) -> None:
        self.outputs.append(lit)

    def ram(self, raddr, waddr, wdata, wbe) -> List[int]:
        """Create a RAM block; returns the 32 rdata literals (new inputs)."""
        rdata = [self.input() for _ in range(RAM_DBITS)]
        self.rams.append(dict(rdata=rdata, raddr=list(raddr), waddr=list(waddr),
                              wdata=list(wdata), wbe=list(wbe)))
        return rdata

    def finish(self) -> Netlist:
        I, L, A = len(self.inputs), len(self.latches), len(self.ands)
        remap = np.zeros(len(self.kind), dtype=np.int64)
        for k, i in enumerate(self.inputs):
            remap[i] = 1 + k
        for k, i in enumerate(self.latches):
            remap[i] = 1 + I + k
        for k, (i, _, _) in enumerate(self.ands):
            remap[i] = 1 + I + L + k

        def m(lit):
            return int(2 * remap[lit >> 1] + (lit & 1))

        for j, n in enumerate(self.latch_next):
            if n is None:
                raise ValueError(f"latch {j} has no next-state")
        rams = []
        for r in self.rams:
            rams.append(RamBlock(rdata=[self.kind[x >> 1][1] for x in r["rdata"]],
                                 raddr=[m(x) for x in r["raddr"]], waddr=[m(x) for x in r["waddr"]],
                                 wdata=[m(x) for x in r["wdata"]], wbe=[m(x) for x in r["wbe"]]))
        return Netlist(
            n_inputs=I,
            latch_next=np.array([m(x) for x in self.latch_next], dtype=np.uint64),
            latch_init=np.array(self.latch_init, dtype=np.uint8),
            outputs=np.array([m(x) for x in self.outputs], dtype=np.uint64),
            and_rhs0=np.array([m(a) for _, a, _ in self.ands], dtype=np.uint64),
            and_rhs1=np.array([m(b) for _, _, b in self.ands], dtype=np.uint64),
            rams=rams, name=self.name)
