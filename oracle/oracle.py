"""ctypes wrapper around oracle.cpp -- TEST INFRASTRUCTURE ONLY (see __init__)."""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build_oracle(force: bool = False) -> str:
    """Compile oracle.cpp with plain g++ -O2 (no -march=native: the .so travels)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build_oracle()
            lib = ctypes.CDLL(_LIB)
            P = ctypes.c_void_p
            u64 = ctypes.c_uint64
            lib.orc_load.restype = P
            lib.orc_load.argtypes = [ctypes.c_char_p]
            lib.orc_last_error.restype = ctypes.c_char_p
            lib.orc_free.argtypes = [P]
            lib.orc_info.argtypes = [P, P]
            lib.orc_reset.argtypes = [P]
            lib.orc_get_state.argtypes = [P, P]
            lib.orc_set_state.argtypes = [P, P]
            lib.orc_get_ram.argtypes = [P, ctypes.c_uint32, P]
            lib.orc_set_ram.argtypes = [P, ctypes.c_uint32, P]
            lib.orc_get_rd.argtypes = [P, P]
            lib.orc_run.argtypes = [P, P, u64, P, P, P, P]
            lib.orc_run_mt.argtypes = [P, P, u64, P, ctypes.c_uint32, P]
            lib.orc_lanes_reset.argtypes = [P, u64]
            lib.orc_lanes_run.argtypes = [P, u64, u64, P, u64, P, P, P]
            lib.orc_lanes_get_state.argtypes = [P, u64, u64, P]
            lib.orc_lanes_get_ram.argtypes = [P, u64, u64, ctypes.c_uint32, P]
            lib.orc_lanes_set_ram.argtypes = [P, u64, u64, ctypes.c_uint32, P]
            lib.orc_digest.argtypes = [P, u64]
            lib.orc_digest.restype = u64
            _lib = lib
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def oracle_digest(words: np.ndarray) -> int:
    w = np.ascontiguousarray(words, dtype=np.uint32)
    return int(_load().orc_digest(_ptr(w), len(w)))


class Oracle:
    """One parsed netlist + simulation state (single stream, plus 64-lane groups)."""

    def __init__(self, path: str):
        lib = _load()
        h = lib.orc_load(path.encode())
        if not h:
            raise ValueError("oracle: " + lib.orc_last_error().decode())
        self._h = h
        self._lib = lib
        info = np.zeros(8, np.uint64)
        lib.orc_info(h, _ptr(info))
        self.n_inputs, self.n_latches, self.n_outputs, self.n_ands, self.n_pi, self.n_rams, self.max_var = \
            (int(x) for x in info[:7])
        self.pi_words = (self.n_pi + 31) // 32
        self.po_words = (self.n_outputs + 31) // 32
        self.q_words = (self.n_latches + 31) // 32
        self.last_seconds = 0.0

    def __del__(self):
        h = getattr(self, "_h", None)
        if h:
            self._lib.orc_free(h)
            self._h = None

    def reset(self):
        self._lib.orc_reset(self._h)

    def get_state(self) -> np.ndarray:
        out = np.zeros(self.q_words, np.uint32)
        self._lib.orc_get_state(self._h, _ptr(out))
        return out

    def set_state(self, words: np.ndarray):
        w = np.ascontiguousarray(words, dtype=np.uint32)
        assert len(w) == self.q_words
        self._lib.orc_set_state(self._h, _ptr(w))

    def get_ram(self, r: int) -> np.ndarray:
        out = np.zeros(8192, np.uint32)
        if self._lib.orc_get_ram(self._h, r, _ptr(out)):
            raise ValueError(self._lib.orc_last_error().decode())
        return out

    def set_ram(self, r: int, words: np.ndarray):
        w = np.ascontiguousarray(words, dtype=np.uint32)
        assert len(w) == 8192
        if self._lib.orc_set_ram(self._h, r, _ptr(w)):
            raise ValueError(self._lib.orc_last_error().decode())

    def get_rd(self) -> np.ndarray:
        out = np.zeros(max(1, self.n_rams), np.uint32)
        self._lib.orc_get_rd(self._h, _ptr(out))
        return out[:self.n_rams]

    def run(self, stim: np.ndarray, po: bool = True, state: bool = False, digest: bool = False):
        """stim uint32[cycles][pi_words] -> dict(po=[cycles][po_words], state=..., digest=...)."""
        stim = np.ascontiguousarray(stim, dtype=np.uint32)
        cycles = stim.shape[0]
        assert stim.shape[1] == self.pi_words, (stim.shape, self.pi_words)
        out = {}
        po_a = np.zeros((cycles, self.po_words), np.uint32) if po else None
        st_a = np.zeros((cycles, self.q_words), np.uint32) if state else None
        dg_a = np.zeros(cycles, np.uint64) if digest else None
        secs = ctypes.c_double(0)
        rc = self._lib.orc_run(self._h, _ptr(stim), cycles, _ptr(po_a), _ptr(st_a), _ptr(dg_a),
                               ctypes.byref(secs))
        if rc:
            raise RuntimeError(self._lib.orc_last_error().decode())
        self.last_seconds = secs.value
        if po:
            out["po"] = po_a
        if state:
            out["state"] = st_a
        if digest:
            out["digest"] = dg_a
        return out

    def run_mt(self, stim: np.ndarray, threads: int) -> np.ndarray:
        """Level-parallel variant of run() on `threads` host threads (CPU baseline,
        SURVEY §8(d)); same results.  Returns po [cycles][po_words]."""
        stim = np.ascontiguousarray(stim, dtype=np.uint32)
        cycles = stim.shape[0]
        assert stim.shape[1] == self.pi_words
        po_a = np.zeros((cycles, self.po_words), np.uint32)
        secs = ctypes.c_double(0)
        if self._lib.orc_run_mt(self._h, _ptr(stim), cycles, _ptr(po_a), threads, ctypes.byref(secs)):
            raise RuntimeError(self._lib.orc_last_error().decode())
        self.last_seconds = secs.value
        return po_a

    # ---- 64-lane batched streams -------------------------------------------
    def lanes_reset(self, groups: int):
        self._lib.orc_lanes_reset(self._h, groups)
        self.n_groups = groups

    def lanes_run(self, group: int, stim: np.ndarray, po: bool = True, digest: bool = False):
        """stim uint32[lanes<=64][cycles][pi_words] for one 64-lane group."""
        stim = np.ascontiguousarray(stim, dtype=np.uint32)
        lanes, cycles, pw = stim.shape
        assert pw == self.pi_words and 1 <= lanes <= 64
        po_a = np.zeros((lanes, cycles, self.po_words), np.uint32) if po else None
        dg_a = np.zeros((lanes, cycles), np.uint64) if digest else None
        secs = ctypes.c_double(0)
        rc = self._lib.orc_lanes_run(self._h, group, lanes, _ptr(stim), cycles, _ptr(po_a), _ptr(dg_a),
                                     ctypes.byref(secs))
        if rc:
            raise RuntimeError(self._lib.orc_last_error().decode())
        self.last_seconds = secs.value
        out = {}
        if po:
            out["po"] = po_a
        if digest:
            out["digest"] = dg_a
        return out

    def lanes_get_state(self, group: int, lane: int) -> np.ndarray:
        out = np.zeros(self.q_words, np.uint32)
        self._lib.orc_lanes_get_state(self._h, group, lane, _ptr(out))
        return out

    def lanes_get_ram(self, group: int, lane: int, r: int) -> np.ndarray:
        out = np.zeros(8192, np.uint32)
        if self._lib.orc_lanes_get_ram(self._h, group, lane, r, _ptr(out)):
            raise ValueError(self._lib.orc_last_error().decode())
        return out

    def lanes_set_ram(self, group: int, lane: int, r: int, words: np.ndarray):
        w = np.ascontiguousarray(words, dtype=np.uint32)
        assert len(w) == 8192
        if self._lib.orc_lanes_set_ram(self._h, group, lane, r, _ptr(w)):
            raise ValueError(self._lib.orc_last_error().decode())
