"""Warp-stall samples of an .ncu-rep source page summed over line ranges.
    python scripts/ncu_line_groups.py rep.ncu-rep name:lo-hi [name:lo-hi ...]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
hdr = rows[h]
si = hdr.index("Warp Stall Sampling (All Samples)")
ii = hdr.index("Instructions Executed")
lines = {}
for r in rows[h + 1:]:
    if len(r) > si and r[0].isdigit():
        lines[int(r[0])] = (int(r[si] or 0), int(r[ii] or 0))
tot = sum(v[0] for v in lines.values()) or 1
for g in sys.argv[2:]:
    name, rng = g.split(":")
    lo, hi = map(int, rng.split("-"))
    s = sum(v[0] for k, v in lines.items() if lo <= k <= hi)
    n = sum(v[1] for k, v in lines.items() if lo <= k <= hi)
    print(f"{name:24s} {100 * s / tot:5.1f}% samples  {n:8d} warp instrs")
