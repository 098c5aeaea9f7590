"""ctypes wrapper of the CPU ISA interpreter (test tool, see isa_interp.cpp)."""
import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "isa_interp.cpp")
LIB = os.path.join(HERE, "libisa.so")
HDR = os.path.join(HERE, "..", "..", "paper_conf_dac_guozwlr25_b200", "csrc", "gem_isa.h")
_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(SRC), os.path.getmtime(HDR)):
            tmp = LIB + f".tmp{os.getpid()}"
            subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", tmp, SRC])
            os.replace(tmp, LIB)
        lib = ctypes.CDLL(LIB)
        P = ctypes.c_void_p
        lib.isa_load.restype = P
        lib.isa_load.argtypes = [P, ctypes.c_size_t]
        lib.isa_free.argtypes = [P]
        lib.isa_run.argtypes = [P, P, ctypes.c_uint64, P, P]
        lib.isa_run_lanes.argtypes = [P, P, ctypes.c_uint64, P, P]
        lib.isa_run_words.argtypes = [P, P, ctypes.c_uint64, P, P]
        lib.isa_last_error.restype = ctypes.c_char_p
        _lib = lib
    return _lib


class IsaInterp:
    def __init__(self, blob: bytes):
        lib = _load()
        self._buf = ctypes.create_string_buffer(blob, len(blob))
        self._h = lib.isa_load(self._buf, len(blob))
        if not self._h:
            raise ValueError(lib.isa_last_error().decode())
        self.lib = lib
        w = np.frombuffer(blob, np.uint32)
        self.n_po, self.n_flops, self.pi_words = int(w[3]), int(w[4]), int(w[10])

    def __del__(self):
        if getattr(self, "_h", None):
            self.lib.isa_free(self._h)

    def run(self, stim, words: bool = False):
        """Bit-packed layers (default) or the word programs (WRD1) of the blob."""
        stim = np.ascontiguousarray(stim, np.uint32)
        T = stim.shape[0]
        po = np.zeros((T, (self.n_po + 31) // 32), np.uint32)
        q = np.zeros((T, (self.n_flops + 31) // 32), np.uint32)
        rc = (self.lib.isa_run_words if words else self.lib.isa_run)(self._h, stim.ctypes.data_as(ctypes.c_void_p), T,
                              po.ctypes.data_as(ctypes.c_void_p), q.ctypes.data_as(ctypes.c_void_p))
        if rc:
            raise RuntimeError(self.lib.isa_last_error().decode())
        return po, q

    def run_lanes(self, stim32):
        """stim32 uint32 [32][cycles][pi_words] -> (po [32][cycles][..], q [32][cycles][..]) via lane programs."""
        stim32 = np.ascontiguousarray(stim32, np.uint32)
        T = stim32.shape[1]
        po = np.zeros((32, T, (self.n_po + 31) // 32), np.uint32)
        q = np.zeros((32, T, (self.n_flops + 31) // 32), np.uint32)
        rc = self.lib.isa_run_lanes(self._h, stim32.ctypes.data_as(ctypes.c_void_p), T,
                                    po.ctypes.data_as(ctypes.c_void_p), q.ctypes.data_as(ctypes.c_void_p))
        if rc:
            raise RuntimeError(self.lib.isa_last_error().decode())
        return po, q
