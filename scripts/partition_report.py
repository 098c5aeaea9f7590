"""Partitioning diagnostics (§III-C):
replication cost vs partition count (the P:107 analogue: RepCut's cost rises
with the partition count), one vs two stages (one extra stage cut the
cost from >200% to <3% at 216 blocks), the effect of the km1 min-cut
refinement, and the effective bit utilisation of the boomerang layers (P:117:
>= 50% after Algorithm 1).  Mapping only (CPU).

usage: python scripts/partition_report.py [c3 [c4]]  -> profiles/r02/partition_report.{json,md}
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_dac_guozwlr25_b200.isa import blob_info  # noqa: E402
from paper_conf_dac_guozwlr25_b200.mapping import compile_file  # noqa: E402
from tests.common import eaig  # noqa: E402


def row(cfg, opts):
    t = time.time()
    i = blob_info(compile_file(eaig(cfg), opts))
    return {"cfg": cfg, "opts": opts, "parts": i.n_parts, "stages": i.n_stages,
            "replication": round(i.replication, 4), "critical_layers": sum(i.stage_max_layers()),
            "total_layers": i.total_layers,
            "slot_util": round(i.n_and_synth / max(1, i.total_layers * 8191), 4),
            "leaf_util": round(i.total_leaves / max(1, i.total_layers * 8192), 4),
            "program_mb": round(i.program_bytes / 1e6, 2), "map_s": round(time.time() - t, 1)}


def main():
    cfgs = sys.argv[1:] or ["c3"]
    rows = []
    for cfg in cfgs:
        counts = [16, 32, 64, 148, 216] if cfg == "c3" else [148, 400]
        for n in counts:
            for stages in (1, 2):
                for km1 in (0, 8):
                    o = f"parts={n} stages={stages} levels=10 key=2 refine=0 merge=0 km1={km1}"
                    r = row(cfg, o)
                    rows.append(r)
                    print(json.dumps(r), flush=True)
    out = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "r02")
    os.makedirs(out, exist_ok=True)
    json.dump(rows, open(os.path.join(out, "partition_report.json"), "w"), indent=1)
    with open(os.path.join(out, "partition_report.md"), "w") as f:
        f.write("# Partitioning diagnostics (mapping only, `scripts/partition_report.py`)\n\n")
        f.write("| cfg | target parts | parts | stages | km1 | replication | critical layers | total layers | "
                "slot util | leaf util | program MB |\n|---|---|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            o = dict(kv.split("=") for kv in r["opts"].split())
            f.write(f"| {r['cfg']} | {o['parts']} | {r['parts']} | {r['stages']} | {o['km1']} | {r['replication']:.3f} | "
                    f"{r['critical_layers']} | {r['total_layers']} | {r['slot_util']:.3f} | {r['leaf_util']:.3f} | "
                    f"{r['program_mb']} |\n")


if __name__ == "__main__":
    main()
