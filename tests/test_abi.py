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


def _load_rc(blob: bytes, n_streams: int = 1):
    """gem_load_program's return code and message (blob validation runs before
    any CUDA call, so this works without a GPU)."""
    from paper_conf_dac_guozwlr25_b200 import gem
    lib = gem.load_library()
    cfg = gem.GemConfig(0, n_streams, None, 0, 0)
    h = ctypes.c_void_p()
    buf = ctypes.create_string_buffer(blob, len(blob))
    rc = lib.gem_load_program(buf, len(blob), ctypes.byref(cfg), ctypes.byref(h))
    return rc, lib.gem_last_error().decode(), h.value


def test_load_program_validates_blob():
    """include/gem.h: a malformed or truncated blob is GEM_E_FORMAT (never an
    out-of-bounds access) and nothing is returned; a well-formed blob passes
    validation (then fails on the missing CUDA device here, GEM_E_UNSUPPORTED,
    or loads on a GPU box)."""
    import numpy as np
    from paper_conf_dac_guozwlr25_b200 import gem
    from tests.common import blob
    b = blob("c1")
    w = np.frombuffer(b, np.uint32).copy()
    rc, msg, h = _load_rc(b)
    if rc == 0:   # GPU box: it loads; free it
        gem.load_library().gem_free(ctypes.c_void_p(h))
    else:
        assert rc == -6 and "CUDA device" in msg, (rc, msg)
    # GH_* word indices of csrc/gem_isa.h
    GH_N_STAGES, GH_OFF_PARTS, GH_OFF_STAGES, GH_OFF_FLOP_INIT, GH_OFF_PROG = 7, 21, 22, 23, 24

    def bad(mut):
        x = w.copy()
        mut(x)
        rc, msg, h = _load_rc(x.tobytes())
        assert h is None
        return rc, msg

    assert bad(lambda x: x.__setitem__(0, 0))[0] == -2                           # magic
    rc, msg = _load_rc(w[:-4].tobytes())[:2]
    assert rc == -2 and "truncated" in msg                                        # size != header
    assert bad(lambda x: x.__setitem__(GH_OFF_PARTS, len(x) - 2))[0] == -2        # part table out of range
    assert bad(lambda x: x.__setitem__(GH_N_STAGES, 0))[0] == -2                  # no stage
    assert bad(lambda x: x.__setitem__(GH_OFF_FLOP_INIT, len(x)))[0] == -2        # permutation tables
    assert bad(lambda x: x.__setitem__(x[GH_OFF_STAGES] + 1, 99))[0] == -2        # stage prefix > n_parts
    assert bad(lambda x: x.__setitem__(x[GH_OFF_PARTS] + 1, 1 << 30))[0] == -2    # program offset
    po = int(w[GH_OFF_PROG] + w[w[GH_OFF_PARTS] + 1])                            # partition 0 program
    assert bad(lambda x: x.__setitem__(po + 14, 300))[0] in (-2, -6)              # chunk count
    assert bad(lambda x: x.__setitem__(po, 0))[0] == -2                           # partition magic
    cfg0 = _load_rc(b, n_streams=0)[0]
    assert cfg0 == -1                                                             # n_streams = 0
