"""Warp-stall samples per SASS instruction from an ncu report (source page).

usage: python scripts/ncu_stalls.py report.ncu-rep [top_n] [--window A:B]
Prints the hottest instructions with their dominant stall reasons, and the
whole SASS listing with sample counts for a window of instruction indices.
"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 40
win = None
if "--window" in sys.argv:
    a, b = sys.argv[sys.argv.index("--window") + 1].split(":")
    win = (int(a), int(b))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
lines = out.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"Address"'))
rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
reasons = [k for k in rows[0] if k.startswith("stall_") and "Not Issued" not in k]
tot = sum(int(r["Warp Stall Sampling (All Samples)"] or 0) for r in rows)
print(f"{len(rows)} SASS instructions, {tot} samples")
agg = {k: sum(int(r[k] or 0) for r in rows) for k in reasons}
print("overall:", ", ".join(f"{k[6:]} {v / tot:.1%}" for k, v in sorted(agg.items(), key=lambda x: -x[1])[:8]))


def fmt(i, r):
    s = int(r["Warp Stall Sampling (All Samples)"] or 0)
    rs = sorted(((int(r[k] or 0), k[6:]) for k in reasons), reverse=True)[:3]
    why = " ".join(f"{n}:{v}" for v, n in rs if v)
    return f"{i:5d} {s:6d} {s / tot:6.1%}  {r['Source'].strip()[:60]:60s} {why}"


order = sorted(range(len(rows)), key=lambda i: -int(rows[i]["Warp Stall Sampling (All Samples)"] or 0))
for i in order[:top]:
    print(fmt(i, rows[i]))
if win:
    print("---- window")
    for i in range(win[0], min(win[1], len(rows))):
        print(fmt(i, rows[i]))

if "--count" in sys.argv:
    # executed warp-instructions per SASS index range (to attribute code regions)
    ex = [int(r["Instructions Executed"] or 0) for r in rows]
    print("total warp-instructions executed:", sum(ex))
    step = int(sys.argv[sys.argv.index("--count") + 1])
    for a in range(0, len(rows), step):
        n = sum(ex[a:a + step])
        smp = sum(int(r["Warp Stall Sampling (All Samples)"] or 0) for r in rows[a:a + step])
        if n or smp:
            print(f"  [{a:5d},{a + step:5d}) inst {n:10d}  samples {smp:6d}  first: {rows[a]['Source'].strip()[:50]}")
