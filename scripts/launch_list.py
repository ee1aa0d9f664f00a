"""Per-launch list (in order) from an ncu --csv launch list: name, grid, us.
    python scripts/launch_list.py launches.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
i = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
hdr, data = rows[i], rows[i + 1:]
kn, mn, mv, idc = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
mu = hdr.index("Metric Unit")
gi = hdr.index("Grid Size") if "Grid Size" in hdr else None
per = collections.OrderedDict()
for r in data:
    d = per.setdefault(r[idc], {"name": r[kn].split("(")[0].replace("void ", ""), "grid": r[gi] if gi else ""})
    if r[mn] == "gpu__time_duration.sum":
        v = float(r[mv].replace(",", ""))
        d["us"] = v / 1e3 if r[mu] in ("ns", "nsecond") else (v * 1e3 if r[mu] in ("ms", "msecond") else v)
tot = 0.0
for lid, d in per.items():
    tot += d.get("us", 0.0)
    print(f"{lid:>5s} {d.get('us', 0.0):9.2f} us  {d['grid']:>14s}  {d['name'][:90]}")
print(f"total {tot:.1f} us over {len(per)} launches")
