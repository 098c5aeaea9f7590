"""Row f3 measurement (GEM_F_ACTIVITY): cycles/s with and without
activity-based partition pruning on
  * gmods  -- tests/circuits.py gated_modules(): 64 modules of depth-48 random
              logic (576K live ANDs), each loading its flops only while its
              enable PI is 1; enables in bursts of 8 every 64 cycles;
  * gmods/aligned -- the same bursts, all enables in phase (the whole design
              idles 56 of every 64 cycles);
  * gmods/random -- the same design with enables Bern(1/2) (little to skip);
  * c3     -- the headline design with its random stimulus (nothing to skip:
              the overhead of the port compare).
Each run is also checked against the oracle (PO trace, first 300 cycles) and
against the run without the flag (whole trace).  One JSON line per run.

usage: python scripts/activity_bench.py [--cycles 2000]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from gen.stimulus import stim_bursts, stimulus  # noqa: E402
from oracle import Oracle  # noqa: E402  (parity check only)
from paper_conf_dac_guozwlr25_b200 import gem  # noqa: E402
from paper_conf_dac_guozwlr25_b200.mapping import compile_file  # noqa: E402
from tests import circuits  # noqa: E402
from tests.common import CACHE, MAP_OPTS, blob, eaig  # noqa: E402


def timed(b, st, flags, reps=3):
    sim = gem.Simulator(b, flags=flags)
    T = st.shape[0]
    sim.set_inputs(st[:min(T, 200)])
    sim.step(min(T, 200))                       # warm-up launch
    best = None
    for _ in range(reps):
        s2 = gem.Simulator(b, flags=flags)
        s2.set_inputs(st)
        s2.step(T)
        ms = s2.last_step_ms()
        po = s2.read_outputs(T)[0]
        act = s2.read_activity() if flags & gem.GEM_F_ACTIVITY else None
        if best is None or ms < best[0]:
            best = (ms, po, act)
        s2.close()
    sim.close()
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cycles", type=int, default=2000)
    a = ap.parse_args()
    T = a.cycles
    os.makedirs(CACHE, exist_ok=True)
    gp = os.path.join(CACHE, "gmods.aag")
    if not os.path.exists(gp):
        circuits.save(circuits.gated_modules(), CACHE, "gmods")
    runs = [("gmods", gp, compile_file(gp, "parts=64"), stim_bursts(64, T, 17)),
            ("gmods/aligned", gp, compile_file(gp, "parts=64"), stim_bursts(64, T, 17, aligned=True)),
            ("gmods/random", gp, compile_file(gp, "parts=64"),
             np.random.default_rng(5).integers(0, 1 << 32, size=(T, 2), dtype=np.uint64).astype(np.uint32)),
            ("c3", eaig("c3"), blob("c3", MAP_OPTS["c3"]), stimulus("c3", 256, T))]
    for name, path, b, st in runs:
        ms0, po0, _ = timed(b, st, 0)
        ms1, po1, act = timed(b, st, gem.GEM_F_ACTIVITY)
        ref = Oracle(path).run(st[:300])["po"]
        ok = bool(np.array_equal(po0, po1) and np.array_equal(po1[:300], ref))
        ev, sk = act
        print(json.dumps({"workload": name, "cycles": T, "cycles_per_s_off": T / ms0 * 1e3,
                          "cycles_per_s_on": T / ms1 * 1e3, "speedup": ms0 / ms1,
                          "partition_cycles_evaluated": ev, "partition_cycles_skipped": sk,
                          "skipped_frac": sk / max(1, ev + sk), "parity_vs_off_and_oracle": ok}), flush=True)


if __name__ == "__main__":
    main()
