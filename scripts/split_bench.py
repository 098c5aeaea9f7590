"""Row f4 on ONE GPU: the cost of the split-design protocol (peer stores of
every committed word + the cross-device barrier) with the ranks emulated as
in-process handles on cuda:0, each on its share of the SMs (grid_limit =
SMs / world).  Not a multi-GPU number: peer memory is local here, so NVLink
latency (~1-2 us per barrier round trip) is not in it; it isolates what the
protocol costs in the kernel.

  python scripts/split_bench.py [--workload c3] [--worlds 1,2,4] [--cycles 1000] [--steps 5]

Prints one JSON line per world: cycles/s (max over the ranks' kernel times),
parity of rank 0's PO trace vs the single-rank run.
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c3")
    ap.add_argument("--worlds", default="1,2,4")
    ap.add_argument("--cycles", type=int, default=1000)
    ap.add_argument("--steps", type=int, default=5)
    args = ap.parse_args()
    import torch
    from gen import stimulus
    from paper_conf_dac_guozwlr25_b200 import gem
    from paper_conf_dac_guozwlr25_b200.dist import connect_local, step_local
    from paper_conf_dac_guozwlr25_b200.isa import blob_info
    from tests.common import blob
    cfg, C = args.workload, args.cycles
    b = blob(cfg)
    info = blob_info(b)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    stims = [stimulus(cfg, info.n_pi, C, seed=103 + k) for k in range(args.steps + 2)]
    ref_po = None
    for world in [int(x) for x in args.worlds.split(",")]:
        if world == 1:
            sims = [gem.Simulator(b, flags=gem.GEM_F_ASYNC)]
        else:
            sims = [gem.Simulator(b, flags=gem.GEM_F_ASYNC, grid_limit=sms // world, dist_world=world, dist_rank=r)
                    for r in range(world)]
            connect_local(sims, C)
        ms, po0 = [], None
        for k in range(args.steps + 2):
            for s in sims:
                s.set_inputs(stims[k])
            t = step_local(sims, C) if world > 1 else [sims[0].step(C) or sims[0].last_step_ms()]
            if k == 0:
                po0 = sims[0].read_outputs(C)
            if k >= 2:
                ms.append(max(t))
        if world == 1:
            ref_po = po0
        own = gem.dist_owner(b, world) if world > 1 else np.zeros(info.n_parts, np.uint32)
        line = {"workload": cfg, "world": world, "cycles_per_s": C / (np.mean(ms) / 1e3),
                "us_per_cycle": np.mean(ms) * 1e3 / C, "grid_per_rank": [s.info["grid"] for s in sims],
                "parts_per_rank": np.bincount(own, minlength=world).tolist(),
                "po_equal_to_world1": bool(ref_po is not None and np.array_equal(po0, ref_po)),
                "note": "ranks emulated in one process on one GPU (peer memory local; no NVLink latency)"}
        print(json.dumps(line), flush=True)
        for s in sims:
            s.close()


if __name__ == "__main__":
    main()
