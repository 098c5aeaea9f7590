"""Run one config for a few cycles (warm-up launch + measured launch) for ncu."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from gen import stimulus  # noqa: E402
from paper_conf_dac_guozwlr25_b200 import gem  # noqa: E402
from tests.common import blob  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--cfg", default="c3")
ap.add_argument("--cycles", type=int, default=50)
ap.add_argument("--streams", type=int, default=1)
ap.add_argument("--launches", type=int, default=2)
a = ap.parse_args()
b = blob(a.cfg)
sim = gem.Simulator(b, n_streams=a.streams)
n_pi = sim.info["n_pi"]
st = np.stack([stimulus("c3" if a.cfg == "c5" else a.cfg, n_pi, a.cycles * a.launches, seed=100 + s)
               for s in range(a.streams)])
sim.set_inputs(st)
for k in range(a.launches):
    sim.step(a.cycles)
    print(f"launch {k}: {sim.last_step_ms():.3f} ms for {a.cycles} cycles "
          f"-> {a.cycles * a.streams / sim.last_step_ms() * 1e3:.0f} stream-cycles/s", flush=True)
print(sim.info)
