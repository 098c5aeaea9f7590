export EXP_CFGS="c5"
python - <<'PY'
import os, subprocess, sys
sys.path.insert(0, '.')
from paper_conf_dac_guozwlr25_b200 import _build
for flags in ["", "-DEXP_LANE_NOCONFLICT"]:
    lib = os.path.join("gpurun_out", f"libgem_{flags.replace('-D','') or 'base'}.so")
    subprocess.check_call([_build.NVCC, *_build.ARCH, "-O3", "-std=c++17", "-shared", "-Xcompiler", "-fPIC", *flags.split(),
                           "-I", "include", "-o", lib, os.path.join(_build.CSRC, "gem_runtime.cu")], stderr=subprocess.DEVNULL)
    out = subprocess.run([sys.executable, "scripts/prof_run.py", "--cfg", "c5", "--cycles", "50", "--streams", "4096", "--phases"],
                         capture_output=True, text=True, env=dict(os.environ, GEM_EXP_LIB=lib))
    print(flags or "base", [l for l in out.stdout.splitlines() if "launch 1" in l or "lane phases" in l], out.stderr[-300:])
PY
