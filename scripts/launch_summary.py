"""Aggregate an ncu --csv launch list: time share and DRAM bytes per kernel."""
import collections
import csv
import sys


def summarise(path):
    rows = list(csv.reader(open(path)))
    i = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr, data = rows[i], rows[i + 1:]
    kn, mn, mv, idc = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
    mu = hdr.index("Metric Unit")
    scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1.0, "us": 1e3, "ms": 1e6,
             "usecond": 1e3, "nsecond": 1.0, "msecond": 1e6}
    per = collections.defaultdict(dict)
    names = {}
    for r in data:
        per[r[idc]][r[mn]] = float(r[mv].replace(",", "")) * scale.get(r[mu], 1.0)
        names[r[idc]] = r[kn].split("(")[0].split("::")[-1].replace("void ", "")
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
    for lid, m in per.items():
        a = agg[names[lid]]
        a[0] += 1
        a[1] += m.get("gpu__time_duration.sum", 0.0)
        a[2] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
    tot = sum(v[1] for v in agg.values())
    out = [f"{'kernel':28s} {'launches':>8s} {'time_ms':>10s} {'share':>6s} {'DRAM_GB':>8s} {'GB/s':>8s}"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        t_ms = v[1] / 1e6 if v[1] > 1e4 else v[1] / 1e3  # ns or us
        out.append(f"{k:28s} {v[0]:8d} {v[1]/1e6:10.3f} {v[1]/tot:6.3f} {v[2]/1e9:8.3f} {v[2]/v[1] if v[1] else 0:8.1f}")
    out.append(f"total device time (serialised, cold) {tot/1e6:.3f} ms over {sum(v[0] for v in agg.values())} launches")
    return "\n".join(out)


if __name__ == "__main__":
    print(summarise(sys.argv[1]))
