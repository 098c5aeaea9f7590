# word_chain A/B: parity on a short window + cycles/s, C1-C3
import sys
sys.path.insert(0, '/root/repo')
import numpy as np
from gen import stimulus
from oracle import Oracle
from paper_conf_dac_guozwlr25_b200 import gem
from tests.common import MAP_OPTS, blob, eaig
for cfg in sys.argv[1:] or ["c1", "c2", "c3"]:
    n_pi = Oracle(eaig(cfg)).n_pi
    T = {"c1": 2000, "c2": 300, "c3": 60}[cfg]
    st = stimulus(cfg, n_pi, max(T, 1000))
    ref = Oracle(eaig(cfg)).run(st[:T], state=True)
    for chain in (1, 2, 3):
        b = blob(cfg, MAP_OPTS[cfg] + f" word_chain={chain}")
        sim = gem.Simulator(b, flags=gem.GEM_F_TRACE_STATE)
        sim.set_inputs(st[:T]); sim.step(T)
        ok = np.array_equal(sim.read_outputs(T)[0], ref["po"]) and np.array_equal(sim.read_state_trace(T)[0], ref["state"])
        s2 = gem.Simulator(b)
        ms = []
        for k in range(4):
            s2.set_inputs(st[:1000]); s2.step(1000); ms.append(s2.last_step_ms())
        print(f"{cfg} chain={chain} words={s2.info['words']} parity={'ok' if ok else 'FAIL'} "
              f"{1000 / np.median(ms[1:]) * 1e3:,.0f} cycles/s", flush=True)
