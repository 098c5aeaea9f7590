"""Word mode (WRD1) quick check: parity vs the oracle on a short window and
cycles/s of word mode vs the bit-packed path on the same blob (one stream)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from gen import stimulus  # noqa: E402
from oracle import Oracle  # noqa: E402
from paper_conf_dac_guozwlr25_b200 import gem  # noqa: E402
from tests.common import MAP_OPTS, blob, eaig  # noqa: E402

cfgs = sys.argv[1:] or ["c1", "c2", "c3"]
for cfg in cfgs:
    opts = MAP_OPTS[cfg] if "words=1" in MAP_OPTS[cfg] else MAP_OPTS[cfg] + " words=1"
    b = blob(cfg, opts)
    n_pi = Oracle(eaig(cfg)).n_pi
    T = {"c1": 2000, "c2": 300, "c3": 60}.get(cfg, 30)
    st = stimulus(cfg, n_pi, max(T, 1000))
    ref = Oracle(eaig(cfg)).run(st[:T], state=True)
    for flags, name in [(0, "words"), (gem.GEM_F_NO_WORDS, "bits")]:
        sim = gem.Simulator(b, flags=flags | gem.GEM_F_TRACE_STATE)
        sim.set_inputs(st[:T])
        sim.step(T)
        po = sim.read_outputs(T)[0]
        q = sim.read_state_trace(T)[0]
        ok = np.array_equal(po, ref["po"]) and np.array_equal(q, ref["state"])
        bad = np.where((po != ref["po"]).any(1) | (q != ref["state"]).any(1))[0][:5]
        sim2 = gem.Simulator(b, flags=flags)
        sim2.set_inputs(st[:1000])
        sim2.step(1000)
        sim2.set_inputs(st[:1000])
        sim2.step(1000)
        ms = sim2.last_step_ms()
        print(f"{cfg} {name:5s} words={sim2.info['words']} grid={sim2.info['grid']} smem={sim2.info['smem_bytes']} "
              f"parity={'ok' if ok else 'FAIL ' + str(bad.tolist())} {1000 / ms * 1e3:,.0f} cycles/s", flush=True)
