"""Debug build with -DGEM_FINE_PROF: per-warp clock64 stamps inside every layer
(up to 32) of cycle 5 on the critical CTA (found by a GEM_F_PROFILE run), next
to the static per-layer statistics of that CTA's partition (leaf-gather LDS,
active warps, leaves).  Stamps: 0 layer start, 1 after gather+fold, 2 next
chunk ready, 3 next records loaded, 4 after top levels, 5 after the barrier;
sub-stamps: gather | fold1 | ballot+fold2 | wo+top.

usage: python scripts/fine_prof.py c3 [map opts]
"""
import ctypes, os, subprocess, sys
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
from paper_conf_dac_guozwlr25_b200 import _build
lib = os.path.join(ROOT, "gpurun_out", "libgem_fine.so")
os.makedirs(os.path.dirname(lib), exist_ok=True)
subprocess.check_call([_build.NVCC, *_build.ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
                       "-DGEM_FINE_PROF", *os.environ.get("FINE_FLAGS", "").split(),
                       "-I", os.path.join(ROOT, "include"), "-o", lib,
                       os.path.join(_build.CSRC, "gem_runtime.cu")])
_build.LIBGEM = lib
_build.build_libgem = lambda force=False, extra=(): lib
from paper_conf_dac_guozwlr25_b200 import gem
from paper_conf_dac_guozwlr25_b200.isa import GP_WORDS
from prog_stats import layer_lds, PH_N_LAYERS, PH_OFF_LAYERS, PH_OFF_CHUNKS
from tests.common import blob
from gen import stimulus

cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
b = blob(cfg, sys.argv[2] if len(sys.argv) > 2 else None)
NL = 32
sim = gem.Simulator(b, flags=gem.GEM_F_PROFILE)
st = stimulus(cfg, sim.info["n_pi"], 50)
sim.set_inputs(st)
sim.step(50)
pr = sim.read_profile().astype(np.int64)
items = (pr[6:40, :, 4] - pr[6:40, :, 0]).mean(0)
crit = int(np.argmax(items))
part = int(pr[5, crit, 10])
print(f"{cfg}: critical CTA {crit} (items {items[crit]:.0f} clk), partition {part}, {pr[5, crit, 6]} layers")
sim.close()
os.environ["GEM_FINE_CTA"] = str(crit)
sim = gem.Simulator(b, flags=gem.GEM_F_PROFILE)
sim.set_inputs(st)
sim.step(50)
out = np.zeros(NL * 96, np.uint64)
sim.lib.gem_read_fine.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
sim.lib.gem_read_fine(sim._h, out.ctypes.data_as(ctypes.c_void_p))
f = out[:NL * 64].reshape(NL, 8, 8).astype(np.int64)     # [layer][warp][slot]
sub = out[NL * 64:].reshape(NL, 8, 4).astype(np.int64)   # [layer][warp][4]
# static stats of the partition's layers
w = np.frombuffer(b, np.uint32)
off_parts, off_prog = int(w[21]), int(w[24])
po = off_prog + int(w[off_parts + part * GP_WORDS + 1])
nl = int(w[po + PH_N_LAYERS])
ctab = w[po + int(w[po + PH_OFF_CHUNKS]):]
L = po + int(w[po + PH_OFF_LAYERS])
stats = []
for l in range(nl):
    n_lds, wf, leaves = layer_lds(w, L)
    stats.append((n_lds, wf, leaves, bin(int(w[L + 1]) & 0xFF).count("1")))
    L += int(ctab[1 + l])
print("layer | total | exec min-max | wait | load | top | bar | gather | fold1 | ballot+fold2 | wo+top || LDS wavefr leaves warps")
tot_all = 0
for l in range(min(nl, NL)):
    if f[l, :, 0].max() == 0:
        break
    d = lambda a, b_: f[l, :, b_] - f[l, :, a]
    ex, wt, ld, tp, br = d(0, 1), d(1, 2), d(2, 3), d(3, 4), d(4, 5)
    tot = f[l, :, 5].max() - f[l, :, 0].min()
    tot_all += tot
    act = sub[l, :, 0] > 0
    g_ = (sub[l, act, 0] - f[l, act, 0]).max() if act.any() else 0
    f1 = (sub[l, act, 1] - sub[l, act, 0]).max() if act.any() else 0
    f2 = (sub[l, act, 2] - sub[l, act, 1]).max() if act.any() else 0
    f3 = (sub[l, act, 3] - sub[l, act, 2]).max() if act.any() else 0
    s_ = stats[l]
    print(f"L{l:2d} | {tot:5d} | {ex.min():4d}-{ex.max():4d} | {wt.max():4d} | {ld.max():4d} | {tp.max():4d} | "
          f"{br.min():4d}-{br.max():4d} | {g_:5d} | {f1:4d} | {f2:4d} | {f3:4d} || {s_[0]:3d} {s_[1]:4d} {s_[2]:5d} {s_[3]}")
print(f"sum of layer totals {tot_all} clk")
