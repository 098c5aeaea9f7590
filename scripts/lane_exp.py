"""Lane-mode timing experiments: run C5 (4096 streams) with libgem variants
built with EXP_LANE_* flags (wrong results on purpose; timing only) and print
launch time + lane phase profile.  Variants are built here (python
scripts/lane_exp.py build FLAGS...) into exp_libs/ and run on the GPU box
(python scripts/lane_exp.py run)."""
import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_dac_guozwlr25_b200 import _build  # noqa: E402

D = os.path.join(ROOT, "exp_libs")
if sys.argv[1] == "build":
    os.makedirs(D, exist_ok=True)
    for flags in sys.argv[2:]:
        tag = flags.replace("-D", "").replace(" ", "_") or "base"
        subprocess.check_call([_build.NVCC, *_build.ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler",
                               "-fPIC", *flags.split(), "-I", os.path.join(ROOT, "include"), "-o",
                               os.path.join(D, f"libgem_{tag}.so"), os.path.join(_build.CSRC, "gem_runtime.cu")])
else:
    cyc = os.environ.get("EXP_CYCLES", "100")
    for rep in range(int(os.environ.get("EXP_REPS", "1"))):
        for lib in sorted(glob.glob(os.path.join(D, "libgem_*.so"))):
            env = dict(os.environ, GEM_EXP_LIB=lib)
            out = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "prof_run.py"), "--cfg", "c5",
                                  "--cycles", cyc, "--streams", "4096", "--phases"], capture_output=True, text=True,
                                 env=env)
            lines = [l for l in out.stdout.splitlines() if "launch 1" in l or "lane phases" in l]
            print(f"[{os.path.basename(lib)}]", *lines, out.stderr[-300:] if out.returncode else "", sep="\n   ",
                  flush=True)
