"""Top CUDA source lines by warp-stall samples from an .ncu-rep (source page)."""
import csv, io, subprocess, sys
rep = sys.argv[1]
skip = sys.argv[2] if len(sys.argv) > 2 else "0"
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
] + ([] if skip == "0" else ["--launch-skip", skip, "--launch-count", "1"]), capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr_i = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
hdr = rows[hdr_i]
si = hdr.index("Warp Stall Sampling (All Samples)")
ii = hdr.index("Instructions Executed")
data = []
for r in rows[hdr_i + 1:]:
    if len(r) <= si or not r[0].isdigit():
        continue
    try:
        data.append((int(r[si] or 0), int(r[ii] or 0), int(r[0]), r[1].strip()[:90]))
    except ValueError:
        pass
tot = sum(d[0] for d in data) or 1
print(f"total samples {tot}")
for s, n, ln, src in sorted(data, reverse=True)[:top]:
    print(f"{100*s/tot:5.1f}% {n:10d} L{ln:4d} {src}")
