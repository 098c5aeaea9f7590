"""A/B timing of libgem builds on one box: time `gem_step` of a config with a
given libgem.so (L2 flushed before every step, median of N steps).

usage: python scripts/ab_time.py <libgem.so> [--cfg c3] [--cycles 1000] [--steps 10] [--streams 1]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("lib")
ap.add_argument("--cfg", default="c3")
ap.add_argument("--cycles", type=int, default=1000)
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--streams", type=int, default=1)
ap.add_argument("--map-opts", default=None)
ap.add_argument("--tune", default="", help="gem_config tuning, e.g. lane_groups=2,lane_ctas_per_sm=2")
a = ap.parse_args()
from paper_conf_dac_guozwlr25_b200 import _build  # noqa: E402
_build.LIBGEM = os.path.abspath(a.lib)
_build.build_libgem = lambda force=False, extra=(): _build.LIBGEM
import torch  # noqa: E402
from gen import stimulus_streams  # noqa: E402
from paper_conf_dac_guozwlr25_b200 import gem  # noqa: E402
from tests.common import blob  # noqa: E402

b = blob(a.cfg, a.map_opts)
tune = {k: (float(v) if k == "l2_evict_last" else int(v)) for k, v in (x.split("=") for x in a.tune.split(",") if x)}
sim = gem.Simulator(b, n_streams=a.streams, **tune)
n_pi = sim.info["n_pi"]
st = stimulus_streams("c5" if a.cfg == "c5" else a.cfg, n_pi, a.cycles, range(a.streams))
flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.int32, device="cuda")
ms = []
for k in range(a.steps + 2):
    flush.fill_(k)
    torch.cuda.synchronize()
    sim.set_inputs(st)
    sim.step(a.cycles)
    if k >= 2:
        ms.append(sim.last_step_ms())
med = float(np.median(ms))
print(f"{os.path.basename(a.lib)} {a.cfg} {a.map_opts or ''}: median {med:.3f} ms / {a.cycles} cycles = "
      f"{a.cycles * a.streams / med * 1e3:.0f} stream-cycles/s (min {min(ms):.3f}, max {max(ms):.3f}) "
      f"grid {sim.info['grid']} layers {sim.info['max_layers']} group {sim.info['group']} {a.tune}", flush=True)
