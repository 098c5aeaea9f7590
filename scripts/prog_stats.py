"""Per-partition / per-layer statistics of a .gemb program: gread size, layers,
leaf-gather modes, padding and shared-memory bank-conflict wavefronts.

usage: python scripts/prog_stats.py c3 [c1 ...]
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_dac_guozwlr25_b200.isa import GP_WORDS, blob_info  # noqa: E402

PH_N_GREAD, PH_N_LAYERS, PH_OFF_LAYERS, PH_OFF_CHUNKS, PH_N_CHUNKS = 1, 2, 7, 13, 14
WM_SPARSE, WM_DENSE, WM_DENSE16 = 0, 1, 2


def wavefronts(words):
    """Shared-memory wavefronts of one LDS over 32 lanes reading u32 `words`."""
    words = np.unique(words)
    return int(np.bincount(words % 32, minlength=32).max())


def layer_lds(w, L):
    """(n_lds, wavefronts, real_leaves, slots) for one layer record at word L."""
    flags = int(w[L + 1])
    n_lds = wf = leaves = 0
    for warp in range(8):
        if not (flags >> warp) & 1:
            continue
        rec = L + int(w[L + 4 + warp])
        mode, n4 = int(w[rec + 4]) & 0xFF, int(w[rec + 4]) >> 8
        lv = w[rec + 136:rec + 136 + 128 * n4].reshape(n4, 32, 4)
        if mode == WM_DENSE16:
            for g in range(n4):
                for k in range(4):
                    e = lv[g, :, k]
                    for half in (e & 0xFFFF, e >> 16):
                        words = (half >> 5) & 0x7FF
                        n_lds += 1
                        wf += wavefronts(words)
                        leaves += int((words != 0).sum())
        else:
            for g in range(n4):
                for k in range(4):
                    words = lv[g, :, k] >> 18
                    n_lds += 1
                    wf += wavefronts(words)
                    leaves += int((lv[g, :, k] != 0).sum())
    return n_lds, wf, leaves


def part_stats(blob):
    w = np.frombuffer(blob, np.uint32)
    info = blob_info(blob)
    off_parts, off_prog = int(w[21]), int(w[24])
    rows = []
    for p in range(info.n_parts):
        po = off_prog + int(w[off_parts + p * GP_WORDS + 1])
        n_gread, nl = int(w[po + PH_N_GREAD]), int(w[po + PH_N_LAYERS])
        ctab = w[po + int(w[po + PH_OFF_CHUNKS]):po + int(w[po + PH_OFF_CHUNKS]) + int(w[po + PH_N_CHUNKS])]
        L = po + int(w[po + PH_OFF_LAYERS])
        tot = np.zeros(3, np.int64)
        for l in range(nl):
            tot += layer_lds(w, L)
            L += int(ctab[1 + l])
        rows.append((p, n_gread, nl, *tot))
    return info, np.array(rows)


if __name__ == "__main__":
    from tests.common import blob
    for cfg in sys.argv[1:] or ["c1", "c3"]:
        info, r = part_stats(blob(cfg))
        crit = r[np.argmax(r[:, 2])]
        print(f"{cfg}: parts={len(r)} layers max={r[:,2].max()} mean={r[:,2].mean():.1f} "
              f"gread mean={r[:,1].mean():.0f} max={r[:,1].max()}")
        print(f"   LDS/layer={r[:,3].sum()/r[:,2].sum():.0f} wavefronts/LDS={r[:,4].sum()/max(1,r[:,3].sum()):.2f} "
              f"leaves/LDS-lane={r[:,5].sum()/max(1,32*r[:,3].sum()):.2f}")
        print(f"   deepest part {crit[0]}: gread={crit[1]} layers={crit[2]} wavefronts/layer={crit[4]/crit[2]:.0f}")
