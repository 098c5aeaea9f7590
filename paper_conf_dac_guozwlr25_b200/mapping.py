"""Python binding of the native mapper (libgemmap.so): E-AIG -> `.gemb` blob.

Argument marshalling only; the mapping flow is C++ (mapper/gem_map.cpp),
as the paper's is native (Rust).
"""
from __future__ import annotations

import ctypes
import threading
from typing import Optional

import numpy as np

from . import _build
from .isa import BlobInfo, blob_info  # noqa: F401

_lib = None
_lock = threading.Lock()


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(_build.build_mapper())
            P = ctypes.c_void_p
            lib.gem_compile.argtypes = [P, ctypes.c_size_t, ctypes.c_char_p, ctypes.POINTER(P),
                                        ctypes.POINTER(ctypes.c_size_t)]
            lib.gem_compile_file.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.POINTER(P),
                                             ctypes.POINTER(ctypes.c_size_t)]
            lib.gem_free_blob.argtypes = [P]
            lib.gem_map_last_error.restype = ctypes.c_char_p
            _lib = lib
    return _lib


def compile_file(path: str, opts: str = "") -> bytes:
    """Map a `.eaig` file; returns the `.gemb` program blob."""
    lib = _load()
    p = ctypes.c_void_p()
    n = ctypes.c_size_t()
    rc = lib.gem_compile_file(path.encode(), opts.encode(), ctypes.byref(p), ctypes.byref(n))
    if rc:
        raise RuntimeError(f"gem_compile failed ({rc}): {lib.gem_map_last_error().decode()}")
    try:
        return ctypes.string_at(p, n.value)
    finally:
        lib.gem_free_blob(p)


def compile_bytes(data: bytes, opts: str = "") -> bytes:
    lib = _load()
    p = ctypes.c_void_p()
    n = ctypes.c_size_t()
    buf = ctypes.create_string_buffer(data, len(data))
    rc = lib.gem_compile(buf, len(data), opts.encode(), ctypes.byref(p), ctypes.byref(n))
    if rc:
        raise RuntimeError(f"gem_compile failed ({rc}): {lib.gem_map_last_error().decode()}")
    try:
        return ctypes.string_at(p, n.value)
    finally:
        lib.gem_free_blob(p)
