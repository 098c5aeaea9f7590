"""Debug build with -DGEM_FINE_PROF: per-warp clock64 stamps inside the first 8
layers of cycle 5 on CTA 0 (0 layer start, 1 after gather+fold, 2 next chunk
ready, 3 next records loaded, 4 after top levels, 5 after the layer barrier)."""
import ctypes, os, subprocess, sys
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_dac_guozwlr25_b200 import _build
lib = os.path.join(ROOT, "gpurun_out", "libgem_fine.so")
os.makedirs(os.path.dirname(lib), exist_ok=True)
subprocess.check_call([_build.NVCC, *_build.ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
                       "-DGEM_FINE_PROF", "-I", os.path.join(ROOT, "include"), "-o", lib,
                       os.path.join(_build.CSRC, "gem_runtime.cu")])
_build.LIBGEM = lib
_build.build_libgem = lambda force=False, extra=(): lib
from paper_conf_dac_guozwlr25_b200 import gem
from tests.common import blob
from gen import stimulus
for cfg in sys.argv[1:] or ["c1"]:
    b = blob(cfg)
    sim = gem.Simulator(b, flags=gem.GEM_F_PROFILE)
    st = stimulus("c3" if cfg == "c5" else cfg, sim.info["n_pi"], 50)
    sim.set_inputs(st)
    sim.step(50)
    out = np.zeros(8 * 8 * 8 + 8 * 8 * 4, np.uint64)
    sim.lib.gem_read_fine.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
    sim.lib.gem_read_fine(sim._h, out.ctypes.data_as(ctypes.c_void_p))
    f = out[:512].reshape(8, 8, 8).astype(np.int64)    # [layer][warp][slot]
    sub = out[512:].reshape(8, 8, 4).astype(np.int64)  # [layer][warp][gather|fold5|ballot+fold5|wo+top]
    print(f"== {cfg} (resident={sim.info.get('resident')}): per-layer, per-warp deltas (clocks): exec | wait_next | load_next | top | barrier")
    for l in range(8):
        if f[l, :, 0].max() == 0:
            break
        d = lambda a, b: f[l, :, b] - f[l, :, a]
        ex, wt, ld, tp, br = d(0, 1), d(1, 2), d(2, 3), d(3, 4), d(4, 5)
        tot = f[l, :, 5].max() - f[l, :, 0].min()
        print(f"  L{l}: total {tot:5d}  exec {ex.min():4d}-{ex.max():4d}  wait {wt.max():4d}  load {ld.max():4d}  "
              f"top {tp.max():4d}  bar {br.min():4d}-{br.max():4d}")
        act = sub[l, :, 0] > 0
        if act.any():
            g_ = sub[l, act, 0] - f[l, act, 0]
            f1 = sub[l, act, 1] - sub[l, act, 0]
            f2 = sub[l, act, 2] - sub[l, act, 1]
            f3 = sub[l, act, 3] - sub[l, act, 2]
            print(f"        active warps {act.sum()}: gather {g_.min()}-{g_.max()}  fold1 {f1.min()}-{f1.max()}  "
                  f"ballot+fold2 {f2.min()}-{f2.max()}  wo+top {f3.min()}-{f3.max()}")
