"""Summarise ncu outputs for profiles/: launch list shares + key metrics of one
--set full capture (dram traffic, duration, IPC, stall reasons, smem wavefronts).

usage: python scripts/ncu_summary.py <launches.csv> <capture.ncu-rep> <out_prefix> [cycles_in_capture]
"""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    agg = defaultdict(lambda: [0, 0.0])
    for d in data:
        k = d["Kernel Name"].split("(")[0]
        agg[k][0] += 1
        agg[k][1] += float(d["Metric Value"])
    tot = sum(v[1] for v in agg.values())
    return [{"kernel": k, "launches": n, "total_ns": t, "share": t / tot, "mean_ns": t / n}
            for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1])]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return dict(zip(r[0], r[2] if len(r) > 2 else r[1])), dict(zip(r[0], r[1]))


def main():
    lc, rep, prefix = sys.argv[1:4]
    cycles = int(sys.argv[4]) if len(sys.argv) > 4 else None
    L = launches(lc) if lc != "-" else []
    d, units = raw(rep)
    kname = d.get("Kernel Name", "kernel").split("(")[0]
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
            "sm__inst_executed.avg.per_cycle_active", "smsp__inst_executed.sum", "launch__grid_size",
            "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
            "smsp__sass_inst_executed_op_shared_ld.sum", "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed"]
    m = {k: (d.get(k), units.get(k)) for k in keys}
    stalls = sorted(((k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""),
                      float(v)) for k, v in d.items()
                     if k.startswith("smsp__average_warps_issue_stalled") and k.endswith("per_issue_active.ratio")),
                    key=lambda t: -t[1])[:8]
    sass = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                          capture_output=True, text=True).stdout
    mn = {k: sass.count(k) for k in ["UBLKCP", "SYNCS.ARRIVE", "SYNCS.PHASECHK", "VOTE.ANY", "SHF.L.W", "LDS.128",
                                     "ATOMG", "UTCHMMA", "HMMA"]}
    res = {"kernel": kname, "launch_list": L, "capture": {k: v[0] for k, v in m.items()}, "capture_units": {k: v[1] for k, v in m.items()},
           "stalls_per_issue": stalls, "sass_mnemonics_in_capture": mn, "capture_cycles": cycles}
    json.dump(res, open(prefix + ".json", "w"), indent=1)
    with open(prefix + ".md", "w") as f:
        f.write("# ncu summary\n\n## Launch list (`--metrics gpu__time_duration.sum --clock-control none`)\n\n")
        f.write("| kernel | launches | mean | share of GPU time |\n|---|---|---|---|\n" if L else
                "(no launch list for this capture)\n")
        for x in L:
            f.write(f"| `{x['kernel']}` | {x['launches']} | {x['mean_ns'] / 1e6:.3f} ms | {x['share']:.4f} |\n")
        f.write(f"\n## `{kname}`, one `--set full` capture\n\n| metric | value | unit |\n|---|---|---|\n")
        for k, (v, u) in m.items():
            f.write(f"| `{k}` | {v} | {u} |\n")
        f.write("\nTop stall reasons (warps stalled per issued instruction):\n\n")
        for k, v in stalls:
            f.write(f"- {k}: {v:.2f}\n")
        f.write("\nSASS evidence in the captured kernel (static counts): " +
                ", ".join(f"`{k}` x{v}" for k, v in mn.items()) + "\n")
    print(open(prefix + ".md").read())


if __name__ == "__main__":
    main()
