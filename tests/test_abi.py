"""C-ABI checks that run without a GPU: libgem.so / libgemmap.so load and
export every function their include/*.h headers declare."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared(header):
    txt = open(os.path.join(ROOT, "include", header)).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(gem_\w+)\s*\(", txt)))


def test_libgem_exports_header():
    from paper_conf_dac_guozwlr25_b200 import _build, gem
    path = _build.build_libgem()
    lib = ctypes.CDLL(path)
    names = _declared("gem.h")
    assert "gem_step" in names and "gem_load_program" in names
    for n in names:
        assert hasattr(lib, n), n
    assert set(gem.EXPORTS) == set(names)


def test_libgemmap_exports_header():
    from paper_conf_dac_guozwlr25_b200 import _build
    lib = ctypes.CDLL(_build.build_mapper())
    for n in _declared("gem_map.h"):
        assert hasattr(lib, n), n


def test_libgem_sm100a_sass():
    """The kernel image is sm_100a SASS (no PTX-only / other-arch fallback)."""
    import shutil
    import subprocess
    from paper_conf_dac_guozwlr25_b200 import _build
    cuobjdump = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(cuobjdump):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([cuobjdump, "--list-elf", _build.build_libgem()], capture_output=True, text=True).stdout
    assert "sm_100a" in out
