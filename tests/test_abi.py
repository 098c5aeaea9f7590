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


def test_load_program_validates_word_programs():
    """Word programs (gem_isa.h WRD1) are bounds-checked on load: an op, output or
    port entry outside the state / its region, a broken step table or a step
    above 1024 ops is GEM_E_FORMAT before any CUDA call."""
    import numpy as np
    from tests.common import blob
    from paper_conf_dac_guozwlr25_b200.isa import GH
    b = blob("c1")
    w = np.frombuffer(b, np.uint32).copy()
    H = {k: i for i, k in enumerate(GH)}
    assert w[H["HAS_WORDS"]] == 1
    wp = int(w[H["OFF_WORD_PROG"]] + w[w[H["OFF_PARTS"]] + 15])    # partition 0's word program
    # WPH_* word indices
    N_GREAD, N_STEPS, N_OPS, N_OUT, STATE, OFF_STEPS, OFF_OPS, OFF_OUT, OFF_GREAD = 1, 2, 3, 4, 6, 7, 8, 9, 11
    ops = wp + int(w[wp + OFF_OPS])
    stp = wp + int(w[wp + OFF_STEPS])
    out = wp + int(w[wp + OFF_OUT])
    gr = wp + int(w[wp + OFF_GREAD])
    lim = int(w[wp + STATE]) * 4

    def rc_of(mut):
        x = w.copy()
        mut(x)
        rc, msg, h = _load_rc(x.tobytes())
        assert h is None
        return rc, msg

    assert rc_of(lambda x: x.__setitem__(wp, 0))[0] == -2                         # magic
    assert rc_of(lambda x: x.__setitem__(ops + 1, lim))[0] == -2                  # op destination
    assert rc_of(lambda x: x.__setitem__(ops + 1, 0))[0] == -2                    # writes word 0
    assert rc_of(lambda x: x.__setitem__(ops, (lim & 0xFFFC) | ((lim & 0xFFFC) << 16)))[0] == -2   # operand
    assert rc_of(lambda x: x.__setitem__(stp + 1, 1 << 20))[0] == -2              # step table
    n_out = int(w[wp + N_OUT])
    assert rc_of(lambda x: x.__setitem__(out, (9 << 24) | 0))[0] == -2            # output region
    assert rc_of(lambda x: x.__setitem__(out + n_out, lim))[0] == -2              # output source
    assert rc_of(lambda x: x.__setitem__(gr, (1 << 24) | (1 << 23)))[0] == -2     # port beyond Q
    assert rc_of(lambda x: x.__setitem__(wp + STATE, 1 << 20))[0] == -2           # state size
