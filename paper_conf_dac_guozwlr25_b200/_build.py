"""In-tree native builds: the mapper (g++) and libgem (nvcc, sm_100a).

Built artefacts live next to their sources so they travel with the repo
snapshot to the GPU box (SURVEY §1 build layers).
"""
from __future__ import annotations

import os
import subprocess
import threading

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
MAPDIR = os.path.join(HERE, "mapper")
LIBMAP = os.path.join(MAPDIR, "libgemmap.so")
LIBGEM = os.path.join(CSRC, "libgem.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
_lock = threading.Lock()


def _stale(out, srcs):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(s) > t for s in srcs)


def _srcs(d, exts):
    return [os.path.join(d, f) for f in sorted(os.listdir(d)) if f.endswith(exts)]


def build_mapper(force: bool = False) -> str:
    srcs = _srcs(MAPDIR, (".cpp", ".h")) + [os.path.join(CSRC, "gem_isa.h")]
    with _lock:
        if force or _stale(LIBMAP, srcs):
            tmp = LIBMAP + f".tmp{os.getpid()}"
            subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", tmp,
                                   os.path.join(MAPDIR, "gem_map.cpp"), "-lpthread"])
            os.replace(tmp, LIBMAP)
    return LIBMAP


def build_libgem(force: bool = False, extra=()) -> str:
    srcs = _srcs(CSRC, (".cu", ".cuh", ".h")) + [os.path.join(os.path.dirname(HERE), "include", "gem.h")]
    with _lock:
        if force or _stale(LIBGEM, srcs):
            tmp = LIBGEM + f".tmp{os.getpid()}"
            cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
                   "-I", os.path.join(os.path.dirname(HERE), "include"), "-o", tmp,
                   os.path.join(CSRC, "gem_runtime.cu"), *extra]
            subprocess.check_call(cmd)
            os.replace(tmp, LIBGEM)
    return LIBGEM
