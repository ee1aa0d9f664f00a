"""Summarise an .ncu-rep: key raw metrics of each captured kernel."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "smsp__inst_executed.sum", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "lts__t_sectors_srcunit_tex_op_read.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "smsp__sass_inst_executed_op_ldgsts.sum"]
STALL = "smsp__average_warps_issue_stalled_"


def summary(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        name = d.get("Kernel Name", "?").split("(")[0]
        lines = [f"kernel {name}"]
        for k in KEYS:
            if k in d:
                lines.append(f"  {k} = {d[k]} {units[hdr.index(k)]}")
        st = sorted(((float(d[k] or 0), k) for k in hdr
                     if k.startswith(STALL) and k.endswith("_per_issue_active.ratio")), reverse=True)
        lines.append("  stalls (per issue): " + ", ".join(
            f"{k[len(STALL):].replace('_per_issue_active.ratio', '')}={v:.2f}" for v, k in st[:7]))
        res.append("\n".join(lines))
    return "\n".join(res)


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(p)
        print(summary(p))
