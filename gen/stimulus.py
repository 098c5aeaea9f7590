"""Seeded stimulus generators (INPUT side only; no circuit arithmetic).

Stimulus layout (shared by the oracle and the C-ABI, `include/gem.h`):
``uint32 [stream][cycle][ceil(n_pi/32)]``; PI i lives in word i/32, bit i%32;
padding bits are 0.  "PI" order = AIGER input order with RAM rdata inputs
removed.  One PI vector per cycle, applied before that cycle's
evaluation (reading U12).

Recipes:
  C1  rst=1 at t in {0,1} and {5000,5001}; en~Bern(3/4); cin~Bern(1/2); a~U32.
  C2  all PIs i.i.d. Bern(1/2).
  C3/C4  PI0 = reset, high for t in {0..3}; other PIs Bern(1/2).
  C5  C3 recipe, stream s seeded with splitmix64(105 ^ s).
"""
from __future__ import annotations

import numpy as np

MASK64 = (1 << 64) - 1


def splitmix64(x: int) -> int:
    x = (x + 0x9E3779B97F4A7C15) & MASK64
    z = x
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def n_words(n_bits: int) -> int:
    return (n_bits + 31) // 32


def pack_bits(bits: np.ndarray) -> np.ndarray:
    """bits[..., n] (0/1) -> uint32[..., ceil(n/32)] little-endian bit order."""
    bits = np.asarray(bits, dtype=np.uint8)
    n = bits.shape[-1]
    nw = n_words(n)
    pad = nw * 32 - n
    if pad:
        bits = np.concatenate([bits, np.zeros(bits.shape[:-1] + (pad,), np.uint8)], -1)
    b = bits.reshape(bits.shape[:-1] + (nw, 32)).astype(np.uint32)
    return (b << np.arange(32, dtype=np.uint32)).sum(-1, dtype=np.uint64).astype(np.uint32)


def unpack_bits(words: np.ndarray, n: int) -> np.ndarray:
    words = np.asarray(words, dtype=np.uint32)
    b = (words[..., None] >> np.arange(32, dtype=np.uint32)) & 1
    b = b.reshape(words.shape[:-1] + (words.shape[-1] * 32,))
    return b[..., :n].astype(np.uint8)


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def stim_c1(cycles: int, seed: int = 1, reset_cycles=(0, 1, 5000, 5001)) -> np.ndarray:
    rng = _rng(seed)
    bits = np.zeros((cycles, 35), np.uint8)
    rc = [t for t in reset_cycles if t < cycles]
    bits[rc, 0] = 1
    bits[:, 1] = rng.random(cycles) < 0.75
    bits[:, 2] = rng.random(cycles) < 0.5
    a = rng.integers(0, 1 << 32, size=cycles, dtype=np.uint64)
    bits[:, 3:] = ((a[:, None] >> np.arange(32, dtype=np.uint64)) & 1).astype(np.uint8)
    return pack_bits(bits)


def stim_random(n_pi: int, cycles: int, seed: int, reset_pi0_cycles: int = 0) -> np.ndarray:
    """Bern(1/2) PIs; PI0 forced to 1 for t < reset_pi0_cycles (then random->0)."""
    rng = _rng(seed)
    nw = n_words(n_pi)
    w = rng.integers(0, 1 << 32, size=(cycles, nw), dtype=np.uint64).astype(np.uint32)
    if n_pi % 32:
        w[:, -1] &= np.uint32((1 << (n_pi % 32)) - 1)
    if reset_pi0_cycles:
        w[:, 0] &= np.uint32(0xFFFFFFFE)
        w[:min(reset_pi0_cycles, cycles), 0] |= np.uint32(1)
    return w


CONFIG_STIM_SEED = {"c1": 1, "c2": 102, "c3": 103, "c4": 104, "c5": 105}


def stimulus(cfg: str, n_pi: int, cycles: int, stream: int = 0, seed: int = None) -> np.ndarray:
    """uint32 [cycles][ceil(n_pi/32)] for one stream of a config."""
    cfg = cfg.lower()
    base = CONFIG_STIM_SEED[cfg] if seed is None else seed
    if cfg == "c1":
        assert n_pi == 35
        return stim_c1(cycles, base)
    if cfg == "c2":
        return stim_random(n_pi, cycles, base)
    if cfg in ("c3", "c4"):
        return stim_random(n_pi, cycles, base, reset_pi0_cycles=4)
    if cfg == "c5":
        s = splitmix64((base ^ stream) & MASK64)
        return stim_random(n_pi, cycles, s, reset_pi0_cycles=4)
    raise ValueError(cfg)


def stimulus_streams(cfg: str, n_pi: int, cycles: int, streams, seed: int = None) -> np.ndarray:
    """uint32 [len(streams)][cycles][ceil(n_pi/32)]."""
    return np.stack([stimulus(cfg, n_pi, cycles, int(s), seed) for s in streams])


def stim_bursts(n_pi: int, cycles: int, seed: int, period: int = 64, duty: int = 8,
                aligned: bool = False) -> np.ndarray:
    """Low-activity stimulus: PI k is 1 only in bursts of `duty` cycles that start
    every `period` cycles at a per-PI random phase (the same phase for every PI
    if `aligned`: the whole design idles between bursts), 0 otherwise (an
    enable per module that is mostly idle).  uint32 [cycles][ceil(n_pi/32)]."""
    rng = _rng(seed)
    nw = n_words(n_pi)
    w = np.zeros((cycles, nw), np.uint32)
    t = np.arange(cycles)
    for k in range(n_pi):
        ph = 0 if aligned else int(rng.integers(period))
        on = ((t + ph) % period) < duty
        w[on, k // 32] |= np.uint32(1 << (k % 32))
    return w


def hold(stim: np.ndarray, r: int) -> np.ndarray:
    """Repeat every input vector r times (inputs that change every r cycles)."""
    return np.repeat(stim, r, axis=-2)
