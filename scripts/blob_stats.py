"""Per-layer statistics of a .gemb program (leaf padding, active warps, write-outs)."""
import sys
import numpy as np
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
from paper_conf_dac_guozwlr25_b200.isa import blob_info, GP_WORDS


def layer_stats(blob):
    w = np.frombuffer(blob, np.uint32)
    info = blob_info(blob)
    off_parts, off_prog = int(w[21]), int(w[24])
    rows = []
    for p in range(info.n_parts):
        po = off_prog + int(w[off_parts + p * GP_WORDS + 1])
        nl = int(w[po + 2])
        L = po + int(w[po + 7])
        for l in range(nl):
            size, flags = int(w[L]), int(w[L + 1])
            active = [(flags >> k) & 1 for k in range(8)]
            leaves = padded = max_lane = lane_wo = dense = 0
            for k in range(8):
                if not active[k]:
                    continue
                rec = L + int(w[L + 4 + k])
                mode, n4 = int(w[rec + 4]) & 0xFF, int(w[rec + 4]) >> 8
                lanes = w[rec + 8:rec + 136].reshape(32, 4)
                lane_wo += int((lanes[:, 3] != 0).sum())
                lv = w[rec + 136:rec + 136 + 128 * n4]
                leaves += int((lv != 0).sum())
                padded += 128 * n4
                max_lane = max(max_lane, 4 * n4)
                dense += mode
            rows.append((p, l, size, sum(active), leaves, padded, max_lane, lane_wo, dense))
            L += size
    return np.array(rows)


if __name__ == "__main__":
    from tests.common import blob
    for cfg in sys.argv[1:] or ["c1", "c2", "c3"]:
        r = layer_stats(blob(cfg))
        print(f"{cfg}: layers={len(r)} words/layer={r[:,2].mean():.0f} active_warps={r[:,3].mean():.2f} "
              f"leaves/layer={r[:,4].mean():.0f} padded/layer={r[:,5].mean():.0f} "
              f"(pad eff {r[:,4].sum()/max(1,r[:,5].sum()):.2f}) max_niter_mean={r[:,6].mean():.1f} "
              f"max_niter_max={r[:,6].max()} thread_wo/layer={r[:,7].mean():.0f} dense_warps/layer={r[:,8].mean():.2f}")
