"""Python binding of libgem (include/gem.h): argument marshalling only.

Every simulation step runs in the sm_100a kernels of csrc/gem_runtime.cu.
There is no CPU fallback: if libgem.so or a CUDA device is missing, the
constructor raises.
"""
from __future__ import annotations

import ctypes
import os
import threading
from typing import Optional

import numpy as np

from . import _build

GEM_F_TRACE_STATE = 0x1
GEM_F_DIGEST = 0x2
GEM_F_ASYNC = 0x4
GEM_F_PROFILE = 0x8
GEM_F_ACTIVITY = 0x10
GEM_F_NO_RESIDENT = 0x20
GEM_F_NO_LANES = 0x40
GEM_F_STATIC_LANES = 0x80
GEM_F_NO_WORDS = 0x100
ERRORS = {-1: "GEM_E_INVAL", -2: "GEM_E_FORMAT", -3: "GEM_E_CUDA", -4: "GEM_E_NOMEM", -5: "GEM_E_NOINPUT",
          -6: "GEM_E_UNSUPPORTED"}
EXPORTS = ["gem_load_program", "gem_info_get", "gem_set_inputs", "gem_step", "gem_read_outputs",
           "gem_read_state", "gem_write_state", "gem_read_state_trace", "gem_read_digests", "gem_read_ram",
           "gem_write_ram", "gem_last_step_ms", "gem_read_profile", "gem_read_activity", "gem_bench_floor", "gem_bench_floor_step", "gem_free", "gem_last_error",
           "gem_dist_owner", "gem_dist_export", "gem_dist_ipc_handles", "gem_dist_ipc_open", "gem_dist_connect"]
GEM_DIST_MAX = 8
GEM_DIST_IPC_BYTES = 328


class GemConfig(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("n_streams", ctypes.c_uint32), ("cuda_stream", ctypes.c_void_p),
                ("flags", ctypes.c_uint32), ("grid_limit", ctypes.c_uint32),
                ("ctas_per_sm", ctypes.c_uint32), ("max_group", ctypes.c_uint32),
                ("lane_groups", ctypes.c_uint32), ("lane_ctas_per_sm", ctypes.c_uint32),
                ("lane_run", ctypes.c_uint32), ("l2_evict_last", ctypes.c_float),
                ("dist_world", ctypes.c_uint32), ("dist_rank", ctypes.c_uint32)]


class GemDistBuffers(ctypes.Structure):
    _fields_ = [(n, ctypes.c_void_p) for n in ("q", "rd", "cut", "po", "flags")] + \
               [("grid", ctypes.c_uint32), ("reserved", ctypes.c_uint32)]


TUNING = ("ctas_per_sm", "max_group", "lane_groups", "lane_ctas_per_sm", "lane_run", "l2_evict_last")


class GemInfo(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint32) for n in
                ("n_pi", "n_po", "n_flops", "n_rams", "n_parts", "n_stages", "max_layers", "total_layers",
                 "pi_words", "po_words", "q_words", "grid", "blocks_per_sm", "smem_bytes", "n_streams",
                 "resident", "ring_slots", "group", "lanes", "words")] + \
               [(n, ctypes.c_uint64) for n in ("n_and", "n_and_mapped", "program_bytes", "cycle")]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n, _ in self._fields_}


class GemError(RuntimeError):
    pass


_lib = None
_lock = threading.Lock()


def library_path() -> str:
    return _build.LIBGEM


def load_library(build: bool = True):
    """Load libgem.so (building it in-tree with nvcc if stale and `build`)."""
    global _lib
    with _lock:
        if _lib is None:
            path = _build.build_libgem() if build else _build.LIBGEM
            if not os.path.exists(path):
                raise GemError(f"libgem.so missing at {path}; there is no CPU fallback")
            lib = ctypes.CDLL(path)
            P = ctypes.c_void_p
            u64 = ctypes.c_uint64
            u32 = ctypes.c_uint32
            lib.gem_load_program.argtypes = [P, ctypes.c_size_t, ctypes.POINTER(GemConfig), ctypes.POINTER(P)]
            lib.gem_info_get.argtypes = [P, ctypes.POINTER(GemInfo)]
            lib.gem_set_inputs.argtypes = [P, P, u64, ctypes.c_int]
            lib.gem_step.argtypes = [P, u64]
            lib.gem_read_outputs.argtypes = [P, P, u64, ctypes.c_int]
            lib.gem_read_state.argtypes = [P, P, ctypes.c_int]
            lib.gem_write_state.argtypes = [P, P, ctypes.c_int]
            lib.gem_read_state_trace.argtypes = [P, P, u64]
            lib.gem_read_digests.argtypes = [P, P, u64]
            lib.gem_read_ram.argtypes = [P, u32, u32, P]
            lib.gem_write_ram.argtypes = [P, u32, u32, P]
            lib.gem_last_step_ms.argtypes = [P, ctypes.POINTER(ctypes.c_float)]
            lib.gem_read_profile.argtypes = [P, P, ctypes.POINTER(u32), ctypes.POINTER(u32)]
            if hasattr(lib, "gem_read_activity"):   # (older builds loaded by A/B timing scripts lack it)
                lib.gem_read_activity.argtypes = [P, ctypes.POINTER(u64), ctypes.POINTER(u64)]
            if hasattr(lib, "gem_dist_connect"):
                DB = ctypes.POINTER(GemDistBuffers)
                lib.gem_dist_owner.argtypes = [P, ctypes.c_size_t, u32, P]
                lib.gem_dist_export.argtypes = [P, u64, DB]
                lib.gem_dist_ipc_handles.argtypes = [P, P]
                lib.gem_dist_ipc_open.argtypes = [P, P, DB]
                lib.gem_dist_connect.argtypes = [P, DB]
            lib.gem_free.argtypes = [P]
            lib.gem_free.restype = None
            lib.gem_last_error.restype = ctypes.c_char_p
            _lib = lib
    return _lib


def _p(a: Optional[np.ndarray]):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def _dev_ptr(t) -> ctypes.c_void_p:
    return ctypes.c_void_p(int(t.data_ptr()))


def dist_owner(blob: bytes, world: int) -> np.ndarray:
    """gem_dist_owner: the rank owning each partition when the design is split
    over `world` devices (host-only, no CUDA call)."""
    lib = load_library()
    n_parts = int(np.frombuffer(blob, np.uint32, count=64)[_GH_N_PARTS])
    out = np.zeros(max(n_parts, 1), np.uint32)
    buf = ctypes.create_string_buffer(blob, len(blob))
    rc = lib.gem_dist_owner(buf, len(blob), world, _p(out))
    if rc != 0:
        raise GemError(f"{ERRORS.get(rc, rc)}: {lib.gem_last_error().decode()}")
    return out[:n_parts]


_GH_N_PARTS = 6   # csrc/gem_isa.h header word


def bench_floor(device: int = 0, grid: int = 148, iters: int = 2000):
    """Latency-floor microbenchmarks (gem_bench_floor): (minimal-layer clocks,
    grid-barrier clocks) measured on `device` with `grid` co-resident CTAs."""
    lib = load_library()
    lib.gem_bench_floor.argtypes = [ctypes.c_int, ctypes.c_uint32, ctypes.c_uint32,
                                    ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]
    a, b = ctypes.c_double(), ctypes.c_double()
    if lib.gem_bench_floor(device, grid, iters, ctypes.byref(a), ctypes.byref(b)) != 0:
        raise GemError(lib.gem_last_error().decode())
    return a.value, b.value


def bench_floor_step(device: int = 0, iters: int = 4000) -> float:
    """Minimal word-mode step clocks (gem_bench_floor_step) measured on `device`."""
    lib = load_library()
    lib.gem_bench_floor_step.argtypes = [ctypes.c_int, ctypes.c_uint32, ctypes.POINTER(ctypes.c_double)]
    a = ctypes.c_double()
    if lib.gem_bench_floor_step(device, iters, ctypes.byref(a)) != 0:
        raise GemError(lib.gem_last_error().decode())
    return a.value


class Simulator:
    """One loaded program on one GPU, with `n_streams` independent stimulus streams."""

    def __init__(self, blob: bytes, device: int = 0, n_streams: int = 1, flags: int = 0,
                 cuda_stream: int = 0, grid_limit: int = 0, dist_world: int = 1, dist_rank: int = 0, **tuning):
        """tuning: gem_config launch-tuning fields (TUNING; 0 = automatic).
        dist_world > 1: this handle is rank `dist_rank` of a design split over
        devices (gem_dist_*; see dist.py) and needs dist_connect before step."""
        self.lib = load_library()
        bad = set(tuning) - set(TUNING)
        if bad:
            raise TypeError(f"unknown gem_config fields {sorted(bad)}")
        cfg = GemConfig(device, n_streams, ctypes.c_void_p(cuda_stream or None), flags, grid_limit)
        cfg.dist_world, cfg.dist_rank = dist_world, dist_rank
        for k, v in tuning.items():
            setattr(cfg, k, v)
        h = ctypes.c_void_p()
        self._blob = ctypes.create_string_buffer(blob, len(blob))
        self._check(self.lib.gem_load_program(self._blob, len(blob), ctypes.byref(cfg), ctypes.byref(h)))
        self._h = h
        self.n_streams = n_streams
        self.flags = flags
        self.info = self.get_info()
        i = self.info
        self.pi_words, self.po_words, self.q_words = i["pi_words"], i["po_words"], i["q_words"]

    def _check(self, rc: int):
        if rc != 0:
            raise GemError(f"{ERRORS.get(rc, rc)}: {self.lib.gem_last_error().decode()}")

    def close(self):
        if getattr(self, "_h", None):
            self.lib.gem_free(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def get_info(self) -> dict:
        out = GemInfo()
        self._check(self.lib.gem_info_get(self._h, ctypes.byref(out)))
        return out.as_dict()

    # ---- inputs / stepping ------------------------------------------------
    def set_inputs(self, pi: np.ndarray):
        """pi: uint32 [n_streams][ncycles][pi_words] (or [ncycles][pi_words] for 1 stream)."""
        pi = np.ascontiguousarray(pi, dtype=np.uint32)
        if pi.ndim == 2:
            pi = pi[None]
        assert pi.shape[0] == self.n_streams and pi.shape[2] == self.pi_words, pi.shape
        self._check(self.lib.gem_set_inputs(self._h, _p(pi), pi.shape[1], 0))

    def set_inputs_device(self, t, ncycles: int):
        """t: torch CUDA uint32/int32 tensor [n_streams][ncycles][pi_words]."""
        self._check(self.lib.gem_set_inputs(self._h, _dev_ptr(t), ncycles, 1))

    def step(self, ncycles: int):
        self._check(self.lib.gem_step(self._h, ncycles))

    # ---- single-design multi-GPU (gem_dist_*) -------------------------------
    def dist_export(self, max_cycles: int) -> GemDistBuffers:
        out = GemDistBuffers()
        self._check(self.lib.gem_dist_export(self._h, max_cycles, ctypes.byref(out)))
        return out

    def dist_ipc_handles(self) -> bytes:
        buf = ctypes.create_string_buffer(GEM_DIST_IPC_BYTES)
        self._check(self.lib.gem_dist_ipc_handles(self._h, buf))
        return buf.raw

    def dist_ipc_open(self, handles: bytes) -> GemDistBuffers:
        assert len(handles) == GEM_DIST_IPC_BYTES
        out = GemDistBuffers()
        buf = ctypes.create_string_buffer(handles, len(handles))
        self._check(self.lib.gem_dist_ipc_open(self._h, buf, ctypes.byref(out)))
        return out

    def dist_connect(self, peers):
        """peers: one GemDistBuffers per rank (this rank's entry is ignored)."""
        arr = (GemDistBuffers * len(peers))(*[p if p is not None else GemDistBuffers() for p in peers])
        self._check(self.lib.gem_dist_connect(self._h, arr))

    def last_step_ms(self) -> float:
        ms = ctypes.c_float()
        self._check(self.lib.gem_last_step_ms(self._h, ctypes.byref(ms)))
        return float(ms.value)

    # ---- outputs ------------------------------------------------------------
    def read_outputs(self, ncycles: int) -> np.ndarray:
        out = np.zeros((self.n_streams, ncycles, self.po_words), np.uint32)
        self._check(self.lib.gem_read_outputs(self._h, _p(out), ncycles, 0))
        return out

    def read_outputs_device(self, t, ncycles: int):
        self._check(self.lib.gem_read_outputs(self._h, _dev_ptr(t), ncycles, 1))

    def read_state(self) -> np.ndarray:
        out = np.zeros((self.n_streams, self.q_words), np.uint32)
        self._check(self.lib.gem_read_state(self._h, _p(out), 0))
        return out

    def write_state(self, q: np.ndarray):
        q = np.ascontiguousarray(q, dtype=np.uint32).reshape(self.n_streams, self.q_words)
        self._check(self.lib.gem_write_state(self._h, _p(q), 0))

    def read_state_trace(self, ncycles: int) -> np.ndarray:
        out = np.zeros((self.n_streams, ncycles, self.q_words), np.uint32)
        self._check(self.lib.gem_read_state_trace(self._h, _p(out), ncycles))
        return out

    def read_digests(self, ncycles: int) -> np.ndarray:
        out = np.zeros((self.n_streams, ncycles), np.uint64)
        self._check(self.lib.gem_read_digests(self._h, _p(out), ncycles))
        return out

    def read_ram(self, ram: int, stream: int = 0) -> np.ndarray:
        out = np.zeros(8192, np.uint32)
        self._check(self.lib.gem_read_ram(self._h, ram, stream, _p(out)))
        return out

    def write_ram(self, ram: int, words: np.ndarray, stream: int = 0):
        w = np.ascontiguousarray(words, dtype=np.uint32)
        assert w.shape == (8192,)
        self._check(self.lib.gem_write_ram(self._h, ram, stream, _p(w)))

    def read_profile(self) -> np.ndarray:
        """uint64 [cycles][grid][16] clock64 phase stamps (GEM_F_PROFILE; slots in include/gem.h)."""
        n, g = ctypes.c_uint32(), ctypes.c_uint32()
        self._check(self.lib.gem_read_profile(self._h, None, ctypes.byref(n), ctypes.byref(g)))
        out = np.zeros((n.value, g.value, 16), np.uint64)
        self._check(self.lib.gem_read_profile(self._h, _p(out), ctypes.byref(n), ctypes.byref(g)))
        return out

    def read_activity(self) -> tuple:
        """(evaluated, skipped) partition-cycles since load (GEM_F_ACTIVITY)."""
        e, k = ctypes.c_uint64(), ctypes.c_uint64()
        self._check(self.lib.gem_read_activity(self._h, ctypes.byref(e), ctypes.byref(k)))
        return int(e.value), int(k.value)

    def run(self, pi: np.ndarray) -> np.ndarray:
        """Convenience: set_inputs + step + read_outputs."""
        pi = np.asarray(pi)
        T = pi.shape[-2]
        self.set_inputs(pi)
        self.step(T)
        return self.read_outputs(T)
