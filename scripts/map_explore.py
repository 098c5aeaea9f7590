"""Explore mapper options: replication, layers, estimated critical-partition cost."""
import sys, time
import numpy as np
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
from paper_conf_dac_guozwlr25_b200.mapping import compile_file
from paper_conf_dac_guozwlr25_b200.isa import blob_info, GP_WORDS
from tests.common import eaig


def part_costs(b):
    i = blob_info(b)
    return np.array(i.part_cost, dtype=np.float64), np.array(i.part_layers)


if __name__ == "__main__":
    cfg = sys.argv[1]
    for opts in sys.argv[2:]:
        t0 = time.time()
        b = compile_file(eaig(cfg), opts)
        i = blob_info(b)
        cost, lay = part_costs(b)
        import heapq
        h = [(0.0, k) for k in range(148)]
        for c in sorted(cost, reverse=True):
            l, k = heapq.heappop(h)
            heapq.heappush(h, (l + c, k))
        mk = max(x[0] for x in h)
        print(f"{opts:40s} LPT148={mk:7.0f} parts={i.n_parts:4d} repl={i.replication:.2f} maxL={i.max_layers:3d} "
              f"meanL={lay.mean():.1f} prog={i.program_bytes/1e6:.1f}MB crit_cost={cost.max():.0f} "
              f"mean_cost={cost.mean():.0f} leaves={i.total_leaves/1e6:.2f}M t={time.time()-t0:.1f}s", flush=True)
