"""Timing experiments: build libgem variants with -D flags and report the phase
profile (per-layer clocks) of c1/c3.  Variants with EXP_* flags compute wrong
results on purpose (they drop parts of a layer) and are never used elsewhere.

usage: python scripts/experiment.py "" "-DEXP_NO_GATHER" ...
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_dac_guozwlr25_b200 import _build  # noqa: E402

cfgs = os.environ.get("EXP_CFGS", "c1 c3").split()
for flags in sys.argv[1:]:
    tag = flags.replace("-D", "").replace(" ", "_") or "base"
    lib = os.path.join(ROOT, "gpurun_out", f"libgem_{tag}.so")
    subprocess.check_call([_build.NVCC, *_build.ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler",
                           "-fPIC", *flags.split(), "-I", os.path.join(ROOT, "include"), "-o", lib,
                           os.path.join(_build.CSRC, "gem_runtime.cu")])
    for cfg in cfgs:
        env = dict(os.environ, GEM_EXP_LIB=lib)
        out = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "prof_run.py"), "--cfg", cfg,
                              "--cycles", "300", "--phases"], capture_output=True, text=True, env=env)
        lines = [l for l in out.stdout.splitlines() if "launch 1" in l or "critical" in l or "all CTAs" in l]
        print(f"[{tag}] {cfg}:", *lines, out.stderr[-300:] if out.returncode else "", sep="\n   ", flush=True)
