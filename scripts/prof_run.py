"""Run one config for a few cycles (warm-up launch + measured launch) for ncu."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from gen import stimulus  # noqa: E402
from paper_conf_dac_guozwlr25_b200 import _build  # noqa: E402
from paper_conf_dac_guozwlr25_b200 import gem  # noqa: E402
from tests.common import blob  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--cfg", default="c3")
ap.add_argument("--cycles", type=int, default=50)
ap.add_argument("--streams", type=int, default=1)
ap.add_argument("--launches", type=int, default=2)
ap.add_argument("--phases", action="store_true")
ap.add_argument("--map-opts", default=None)
a = ap.parse_args()
b = blob(a.cfg, a.map_opts)
sim = gem.Simulator(b, n_streams=a.streams)
n_pi = sim.info["n_pi"]
st = np.stack([stimulus("c3" if a.cfg == "c5" else a.cfg, n_pi, max(200, a.cycles * a.launches), seed=100 + s)
               for s in range(a.streams)])
sim.set_inputs(st)
for k in range(a.launches):
    sim.step(a.cycles)
    print(f"launch {k}: {sim.last_step_ms():.3f} ms for {a.cycles} cycles "
          f"-> {a.cycles * a.streams / sim.last_step_ms() * 1e3:.0f} stream-cycles/s", flush=True)
print(sim.info)

if a.phases:
    psim = gem.Simulator(b, n_streams=a.streams, flags=gem.GEM_F_PROFILE)
    psim.set_inputs(st[:, :200])
    psim.step(200)
    pr = psim.read_profile().astype(np.int64)[20:]     # skip warm-up cycles
    d = lambda a_, b_: (pr[:, :, b_] - pr[:, :, a_])
    gread, layers, out = d(0, 1), d(1, 2), d(2, 3)
    items, bar = d(0, 4), d(4, 5)
    tot = d(0, 5)
    nl = pr[:, :, 6]
    crit = np.argmax(items.mean(0))
    print(f"phases (SM clocks, mean over cycles): cycle total {tot.mean():.0f}")
    print(f"  critical CTA {crit}: layers={nl[0, crit]} gread={gread[:, crit].mean():.0f} "
          f"layers={layers[:, crit].mean():.0f} ({layers[:, crit].mean() / max(1, nl[0, crit]):.0f}/layer) "
          f"out+ram={out[:, crit].mean():.0f} items={items[:, crit].mean():.0f} barrier={bar[:, crit].mean():.0f}")
    c0, grl, l0, gb = d(0, 7), d(7, 8), d(8, 9), d(9, 1)
    print(f"  critical CTA gread split: chunk0 ready {c0[:, crit].mean():.0f}, port loads (thread 0) "
          f"{grl[:, crit].mean():.0f}, layer-0 records {l0[:, crit].mean():.0f}, barrier {gb[:, crit].mean():.0f}")
    if not sim.info.get("lanes"):
        e11 = d(2, 11)
        print(f"  critical CTA commit split: endpoints {e11[:, crit].mean():.0f}, RAM + sync {d(11, 3)[:, crit].mean():.0f}")
    per_layer = layers.mean(0) / np.maximum(1, nl[0])
    print(f"  all CTAs: items mean {items.mean():.0f} max {items.mean(0).max():.0f}; per-layer clocks "
          f"mean {per_layer.mean():.0f} min {per_layer.min():.0f} max {per_layer.max():.0f}; "
          f"gread mean {gread.mean():.0f}; out mean {out.mean():.0f}; barrier min {bar.mean(0).min():.0f}")

if a.phases and sim.info.get("lanes"):
    # lane mode: per-CTA sums over its work items of gread / layers / out / ram clocks (slots 11-14)
    acc = pr[:, :, 11:16].astype(np.float64)
    items_t = (pr[:, :, 4] - pr[:, :, 0]).astype(np.float64)
    bar_t = (pr[:, :, 5] - pr[:, :, 4]).astype(np.float64)
    print(f"lane phases per cycle (mean over CTAs): items {items_t.mean():.0f} clk = chunk0 {acc[:, :, 0].mean():.0f} + "
          f"gread {acc[:, :, 1].mean():.0f} + layer0/sync {acc[:, :, 2].mean():.0f} + layers {acc[:, :, 3].mean():.0f} + "
          f"out+ram {acc[:, :, 4].mean():.0f}; "
          f"barrier {bar_t.mean():.0f}; items max {items_t.mean(0).max():.0f}")
