"""Summarise an `ncu --set full` report: key memory / occupancy metrics and stall reasons per launch.

    python scripts/ncu_summary.py gpurun_out/prof.ncu-rep [more.ncu-rep ...]
"""
import csv
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sectors.sum", "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
    "l1tex__throughput.avg.pct_of_peak_sustained_active", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
    "launch__occupancy_limit_registers", "smsp__inst_executed.sum", "lts__t_sectors_op_atom.sum",
    "lts__t_sectors_op_red.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "smsp__sass_data_bytes_mem_global_op_ld.sum",
    "l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum",
]


def summarise(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    lines = []
    for vals in rows[2:]:
        name = vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        lines.append(f"## {name.split('(')[0]}  (id {vals[hdr.index('ID')] if 'ID' in hdr else '?'})")
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                lines.append(f"  {k:58s} {vals[i]:>22s} {units[i]}")
        try:
            sb = vals[hdr.index("smsp__sass_data_bytes_mem_global_op_ld.sum")]
            ss = vals[hdr.index("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum")]
            eff = float(sb.replace(",", "")) / (32.0 * float(ss.replace(",", "")))
            lines.append(f"  {'LSU sector efficiency (bytes used / 32*sectors)':58s} {eff:22.3f}")
        except Exception:
            pass
        stalls = []
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warps_issue_stalled") and h.endswith("per_issue_active.ratio"):
                try:
                    stalls.append((float(vals[i]), h.replace("smsp__average_warps_issue_stalled_", "")
                                   .replace("_per_issue_active.ratio", "")))
                except ValueError:
                    pass
        lines.append("  top stall reasons (warps stalled per issue): " +
                     ", ".join(f"{n}={v:.2f}" for v, n in sorted(stalls, reverse=True)[:5]))
    return "\n".join(lines)


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(f"# {p}")
        print(summarise(p))
