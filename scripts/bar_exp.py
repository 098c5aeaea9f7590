"""Grid-barrier variants (GEM_BAR_VARIANT) on the floor microbenchmark and c3."""
import os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_dac_guozwlr25_b200 import _build
for v in sys.argv[1:]:
    lib = os.path.join(ROOT, "gpurun_out", f"libgem_bar{v}.so")
    subprocess.check_call([_build.NVCC, *_build.ARCH, "-O3", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
                           f"-DGEM_BAR_VARIANT={v}", "-I", os.path.join(ROOT, "include"), "-o", lib,
                           os.path.join(_build.CSRC, "gem_runtime.cu")], stderr=subprocess.DEVNULL)
    code = ("import sys; sys.path.insert(0, %r)\nfrom paper_conf_dac_guozwlr25_b200 import _build\n"
            "_build.LIBGEM = %r\n_build.build_libgem = lambda force=False, extra=(): _build.LIBGEM\n"
            "from paper_conf_dac_guozwlr25_b200 import gem\nprint('floor', gem.bench_floor(0, 148))" % (ROOT, lib))
    print(f"[variant {v}]", subprocess.run([sys.executable, "-c", code], capture_output=True, text=True).stdout.strip())
    out = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "prof_run.py"), "--cfg", "c3", "--cycles", "500",
                          "--phases"], capture_output=True, text=True, env=dict(os.environ, GEM_EXP_LIB=lib)).stdout
    print("\n".join(l for l in out.splitlines() if "launch 1" in l or "critical CTA 1" in l or "all CTAs" in l), flush=True)
