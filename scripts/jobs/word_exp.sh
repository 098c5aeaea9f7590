# timing experiments (results wrong on purpose): marginal cost of word-mode phases on C3
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for e in 0 1 2 3; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC -DWORD_EXP=$e -I include \
    -o paper_conf_dac_guozwlr25_b200/csrc/libgem.so paper_conf_dac_guozwlr25_b200/csrc/gem_runtime.cu
  python - <<PY
import sys; sys.path.insert(0, '.')
import numpy as np
from gen import stimulus
from paper_conf_dac_guozwlr25_b200 import gem
from tests.common import blob
for cfg in ("c3", "c1"):
    b = blob(cfg); sim = gem.Simulator(b)
    st = stimulus(cfg, sim.info["n_pi"], 1000)
    ms = []
    for k in range(4):
        sim.set_inputs(st); sim.step(1000); ms.append(sim.last_step_ms())
    print("exp $e", cfg, "%.0f cycles/s" % (1000 / np.median(ms[1:]) * 1e3), "clk/cycle %.0f" % (np.median(ms[1:]) * 1e-3 / 1000 * 1965e6))
PY
done
