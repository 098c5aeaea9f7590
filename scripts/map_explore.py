"""Explore mapper options: replication, layers, estimated critical-partition cost."""
import sys, time
import numpy as np
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
from paper_conf_dac_guozwlr25_b200.mapping import compile_file
from paper_conf_dac_guozwlr25_b200.isa import blob_info, GP_WORDS
from tests.common import eaig


def part_costs(b, a=150.0, c=12.0):
    """est. cycles per partition-cycle: sum over layers of a + c * sum_w niter_w / 4 (issue-bound)."""
    w = np.frombuffer(b, np.uint32)
    i = blob_info(b)
    op, opr = int(w[21]), int(w[24])
    costs, layers = [], []
    for p in range(i.n_parts):
        po = opr + int(w[op + p * GP_WORDS + 1])
        nl = int(w[po + 2])
        L = po + int(w[po + 7])
        t = 0.0
        for l in range(nl):
            niter = w[L + 4:L + 12].astype(np.int64)
            t += a + c * max(niter.max(), niter.sum() / 4)
            L += int(w[L])
        costs.append(t)
        layers.append(nl)
    return np.array(costs), np.array(layers)


if __name__ == "__main__":
    cfg = sys.argv[1]
    for opts in sys.argv[2:]:
        t0 = time.time()
        b = compile_file(eaig(cfg), opts)
        i = blob_info(b)
        cost, lay = part_costs(b)
        print(f"{opts:40s} parts={i.n_parts:4d} repl={i.replication:.2f} maxL={i.max_layers:3d} "
              f"meanL={lay.mean():.1f} prog={i.program_bytes/1e6:.1f}MB crit_cost={cost.max():.0f} "
              f"mean_cost={cost.mean():.0f} leaves={i.total_leaves/1e6:.2f}M t={time.time()-t0:.1f}s", flush=True)
