"""Short runs for compute-sanitizer (memcheck / racecheck / synccheck / initcheck),
SURVEY §5: C1, a small RAM + 2-stage design (resident, streamed ring and
multi-item CTAs) and lane mode, each checked bit-exact against the oracle.

usage: compute-sanitizer --tool <tool> python scripts/sanitize_run.py
"""
import os
import sys
import tempfile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from gen import stimulus  # noqa: E402
from gen.stimulus import stim_random  # noqa: E402
from oracle import Oracle  # noqa: E402
from paper_conf_dac_guozwlr25_b200 import gem  # noqa: E402
from paper_conf_dac_guozwlr25_b200.mapping import compile_file  # noqa: E402
from tests import circuits  # noqa: E402
from tests.common import blob, eaig  # noqa: E402


def check(name, b, path, st, n_streams=1, **kw):
    sim = gem.Simulator(b, n_streams=n_streams, **kw)
    T = st.shape[-2]
    sim.set_inputs(st if st.ndim == 3 else st[None])
    sim.step(T)
    po = sim.read_outputs(T)
    stims = st if st.ndim == 3 else st[None]
    o = Oracle(path)
    if n_streams >= 32:
        o.lanes_reset(1)
        r = o.lanes_run(0, stims[:64])
        ok = np.array_equal(po[:64], r["po"])
    else:
        ok = all(np.array_equal(po[s], Oracle(path).run(stims[s])["po"]) for s in range(n_streams))
    print(f"{name}: {'ok' if ok else 'MISMATCH'} ({sim.info['grid']} CTAs, lanes={sim.info['lanes']}, "
          f"words={sim.info['words']})", flush=True)
    sim.close()
    return ok


ok = True
ok &= check("c1 words", blob("c1"), eaig("c1"), stimulus("c1", 35, 60))
ok &= check("c1 bits", blob("c1"), eaig("c1"), stimulus("c1", 35, 60), flags=gem.GEM_F_NO_WORDS)
with tempfile.TemporaryDirectory() as d:
    net = circuits.small_G(seed=21, n_and=3000, with_ram=True)
    p = circuits.save(net, d, "g")
    st = stim_random(net.n_pi, 12, 3, reset_pi0_cycles=2)
    for opts, kw in [("parts=4", {}), ("parts=4 stages=2", {}), ("parts=4", {"grid_limit": 2}),
                     ("parts=4", {"flags": gem.GEM_F_NO_RESIDENT}), ("parts=4 words=1", {}),
                     ("parts=4 stages=2 words=1", {}), ("parts=4 words=1", {"grid_limit": 2}),
                     ("parts=4 words=1", {"grid_limit": 1}), ("parts=1 words=1", {})]:
        ok &= check(f"small {opts} {kw}", compile_file(p, opts), p, st, **kw)
    S = 64
    stl = np.stack([stim_random(net.n_pi, 6, 100 + s, reset_pi0_cycles=2) for s in range(S)])
    ok &= check("lanes", compile_file(p, "parts=3 lanes=1"), p, stl, n_streams=S)
sys.exit(0 if ok else 1)
