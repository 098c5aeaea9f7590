"""Word-mode mapping exploration (CPU only): for each mapper option set, the
critical word program's step widths and an estimated per-cycle step cost
(narrow step ~110 clk, +100 clk per extra 256-op round)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_dac_guozwlr25_b200.isa import blob_info  # noqa: E402
from paper_conf_dac_guozwlr25_b200.mapping import compile_file  # noqa: E402
from tests.common import eaig  # noqa: E402


def est(b):
    w = np.frombuffer(b, np.uint32)
    info = blob_info(b)
    off_w, np_ = int(w[48]), info.n_parts
    pt = w[int(w[21]):int(w[21]) + 16 * np_].reshape(np_, 16)
    worst = (0, None)
    for p in range(np_):
        h = off_w + int(pt[p, 15])
        ns = int(w[h + 2])
        stp = w[h + int(w[h + 7]):h + int(w[h + 7]) + ns + 1].astype(np.int64)
        n = np.diff(stp)
        cost = float(np.sum(110 + 100 * np.maximum(0, (n + 255) // 256 - 1)))
        if cost > worst[0]:
            worst = (cost, n)
    return worst[0], len(worst[1]), int((worst[1] > 256).sum()), info


cfg = sys.argv[1]
for opts in sys.argv[2:]:
    t = time.time()
    b = compile_file(eaig(cfg), opts + " words=1")
    cost, ns, wide, info = est(b)
    print(f"{opts!r}: parts={info.n_parts} repl={info.replication:.2f} steps={ns} wide={wide} est_step_clk={cost:.0f} "
          f"has_words={info.has_words} ({time.time() - t:.0f}s)", flush=True)
