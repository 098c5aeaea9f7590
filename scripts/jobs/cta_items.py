# per-CTA item clocks of a word-mode C3 run (GEM_F_PROFILE): which partitions bind the cycle
import sys
sys.path.insert(0, '/root/repo')
import numpy as np
from gen import stimulus
from paper_conf_dac_guozwlr25_b200 import gem
from paper_conf_dac_guozwlr25_b200.isa import blob_info
from tests.common import blob
cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
b = blob(cfg)
info = blob_info(b)
w = np.frombuffer(b, np.uint32)
off_w = int(w[48]); np_ = info.n_parts
pt = w[int(w[21]):int(w[21]) + 16 * np_].reshape(np_, 16)
ops = {}
for p in range(np_):
    h = off_w + int(pt[p, 15])
    ops[p] = (int(w[h + 3]), int(w[h + 2]))
sim = gem.Simulator(b, flags=gem.GEM_F_PROFILE)
st = stimulus(cfg, sim.info["n_pi"], 200)
sim.set_inputs(st); sim.step(200)
pr = sim.read_profile().astype(np.int64)[20:]
items = (pr[:, :, 4] - pr[:, :, 0]).mean(0)
steps_clk = (pr[:, :, 2] - pr[:, :, 1]).mean(0)
part = pr[0, :, 10]
order = np.argsort(-items)
for i in order[:15]:
    p = int(part[i])
    print(f"cta {i:3d} part {p:3d} items {items[i]:7.0f} steps_clk {steps_clk[i]:7.0f} ops {ops[p][0]:6d} steps {ops[p][1]:3d}")
print("median items", np.median(items))
