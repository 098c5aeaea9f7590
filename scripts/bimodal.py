"""Experiment: is C3's gem_step_kernel duration a property of the simulator
instance (its allocations) or of the run?  Four instances in one process,
timed round-robin with an L2 flush before each step."""
import numpy as np
import torch

import bench
from paper_conf_dac_guozwlr25_b200 import gem
from paper_conf_dac_guozwlr25_b200.isa import blob_info
from tests.common import blob

b = blob("c3")
info = blob_info(b)
C = 1000
x = bench.workload_inputs("c3", info.n_pi, C, [0], 1)
flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.int32, device="cuda")
sims = [gem.Simulator(b, n_streams=1) for _ in range(4)]
res = {i: [] for i in range(4)}
for rnd in range(6):
    for i, s in enumerate(sims):
        flush.fill_(rnd)
        torch.cuda.synchronize()
        s.set_inputs(x)
        s.step(C)
        res[i].append(s.last_step_ms())
for i in range(4):
    print("instance", i, "kernel ms", np.round(res[i][1:], 3).tolist())
