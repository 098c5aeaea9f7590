"""Shared test helpers: cached netlists, blobs and oracle runs (no method arithmetic)."""
from __future__ import annotations

import functools
import zlib
import os

import numpy as np

from gen import netlist_path, stimulus, stimulus_streams

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CACHE = os.environ.get("GEM_CACHE") or os.path.join(ROOT, ".cache")

# mapper options per config (also used by bench.py)
MAP_OPTS = {"c1": "levels=10 words=1", "c2": "levels=10 key=2 part_size=2000 words=1",
            "c3": "part_size=7000 max_parts=148 levels=10 key=2 merge_ratio=0.6 merge_cap=9000 words=1",
            "c4": "stages=1 levels=10 key=2 part_size=22000", "c5": "refine=0 lanes=1 key=2 merge_cap=60000 lane_words=7000 levels=10 merge_ratio=0.5"}


@functools.lru_cache(maxsize=None)
def eaig(cfg: str) -> str:
    return netlist_path(cfg, CACHE)


@functools.lru_cache(maxsize=None)
def blob(cfg: str, opts: str = None) -> bytes:
    from paper_conf_dac_guozwlr25_b200.mapping import compile_file
    o = MAP_OPTS[cfg] if opts is None else opts
    key = f"{cfg}_{zlib.crc32(o.encode()):08x}"
    p = os.path.join(CACHE, key + ".gemb")
    src = eaig(cfg)
    if os.path.exists(p) and os.path.getmtime(p) > os.path.getmtime(src):
        lib = __import__("paper_conf_dac_guozwlr25_b200._build", fromlist=["LIBMAP"]).LIBMAP
        if not os.path.exists(lib) or os.path.getmtime(p) > os.path.getmtime(lib):
            return open(p, "rb").read()
    b = compile_file(src, o)
    tmp = p + f".tmp{os.getpid()}"
    open(tmp, "wb").write(b)
    os.replace(tmp, p)
    return b
