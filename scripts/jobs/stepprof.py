# experiment: per-step clocks of the critical CTA in word mode (temporary debug stamps)
import sys
sys.path.insert(0, '/root/repo')
import numpy as np
from gen import stimulus
from paper_conf_dac_guozwlr25_b200 import gem
from tests.common import blob, MAP_OPTS
cfg = sys.argv[1]
b = blob(cfg)
sim = gem.Simulator(b, flags=gem.GEM_F_PROFILE)
st = stimulus(cfg, sim.info['n_pi'], 200)
sim.set_inputs(st); sim.step(200)
pr = sim.read_profile().astype(np.int64)
G = pr.shape[1]
flat = pr.reshape(-1)
items = (pr[20:, :, 4] - pr[20:, :, 0]).mean(0)
crit = int(np.argmax(items))
base = 5 * G * 16 + crit * 64
stamps = flat[base:base + 64]
t1 = stamps[63]
ns = int(pr[10, crit, 6])
d = np.diff(np.concatenate([[t1], stamps[:ns]]))
print(cfg, "critical CTA", crit, "steps", ns, "sum", int(d.sum()))
print("per-step clk:", d.tolist())
