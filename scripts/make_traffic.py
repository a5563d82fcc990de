"""profiles/traffic.json from an ncu launch list with DRAM metrics of ONE BFS (host-driven loop):

    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
        --csv --log-file launches.csv python scripts/profile_one_bfs.py auto
    python scripts/make_traffic.py launches.csv [push_only_launches.csv] > profiles/traffic.json

Per bench roofline class: mean DRAM bytes (read + write) per advance launch, where one push
advance = k_push_words + k_push_heavy (+ k_push_seg) and one pull advance = k_pull_bfs; from the
optional push-only list, the dense supersteps' sweep (k_push_sweep + k_frontier_arcs)."""
import collections
import csv
import json
import sys


def load(path):
    lines = open(path).read().splitlines()
    start = [i for i, l in enumerate(lines) if l.startswith('"ID"')][0]
    rows = list(csv.reader(lines[start:]))
    hdr = rows[0]
    ki, mi, vi, ii = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
    launches = collections.OrderedDict()
    for r in rows[1:]:
        key = (int(r[ii]), r[ki].split("(")[0].replace("void ", ""))
        launches.setdefault(key, {})[r[mi]] = float(r[vi].replace(",", ""))
    return launches


def main(path, push_path=None):
    launches = load(path)
    # keep the last BFS: from the last k_seed on
    items = list(launches.items())
    last_seed = max(i for i, ((_, k), _) in enumerate(items) if "k_seed" in k)
    items = items[last_seed:]
    push, pull, diff, cur = [], [], [], None
    sect = {"advance_push": [0.0, 0.0], "advance_pull": [0.0, 0.0], "compact": [0.0, 0.0], "advance_sweep": [0.0, 0.0]}

    def add_sect(cls, m):
        sect[cls][0] += m.get("smsp__sass_data_bytes_mem_global_op_ld.sum", 0.0)
        sect[cls][1] += m.get("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", 0.0)
    for (_, k), m in items:
        b = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
        t = m.get("gpu__time_duration.sum", 0.0)
        if "k_push_words" in k:
            cur = [b, t]
            push.append(cur)
            add_sect("advance_push", m)
        elif ("k_push_heavy" in k or "k_push_seg" in k) and cur is not None:
            cur[0] += b
            cur[1] += t
            add_sect("advance_push", m)
        elif "k_pull_bfs" in k:
            pull.append([b, t])
            add_sect("advance_pull", m)
            cur = None
        elif "k_bfs_diff" in k:
            diff.append([b, t])
            add_sect("compact", m)

    def eff(cls):
        by, se = sect[cls]
        return by / (32.0 * se) if se else None
    out = {
        "source": f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum ({path}); "
                  "one DO BFS on config 4, cold-cache serialised launches",
        "advance_push": {"dram_bytes_per_launch": sum(b for b, _ in push) / max(len(push), 1), "launches": len(push),
                         "ncu_ms_total": sum(t for _, t in push) / 1e6},
        "advance_pull": {"dram_bytes_per_launch": sum(b for b, _ in pull) / max(len(pull), 1), "launches": len(pull),
                         "ncu_ms_total": sum(t for _, t in pull) / 1e6},
        "compact": {"dram_bytes_per_launch": sum(b for b, _ in diff) / max(len(diff), 1), "launches": len(diff),
                    "ncu_ms_total": sum(t for _, t in diff) / 1e6},
    }
    for cls in ("advance_push", "advance_pull", "compact"):
        out[cls]["lsu_sector_efficiency"] = eff(cls)
    out["sector_efficiency_def"] = ("smsp__sass_data_bytes_mem_global_op_ld / (32 x l1tex__t_sectors_pipe_lsu_mem_global_op_ld) "
                                    "over the class's launches (LSU loads only; TMA bulk copies bypass the LSU pipe)")
    if push_path:
        sw = []
        for (_, k), m in load(push_path).items():
            b = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
            t = m.get("gpu__time_duration.sum", 0.0)
            if "k_push_sweep" in k:
                sw.append([b, t, m.get("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed")])
                add_sect("advance_sweep", m)
            elif "k_frontier_arcs" in k and sw:
                sw[-1][0] += b
                sw[-1][1] += t
        heavy = max(sw, key=lambda x: x[1]) if sw else None
        out["advance_sweep"] = {
            "source": f"ncu launch list of one push-only BFS ({push_path})",
            "dram_bytes_per_launch": sum(b for b, _, _ in sw) / max(len(sw), 1), "launches": len(sw),
            "ncu_ms_total": sum(t for _, t, _ in sw) / 1e6,
            "ncu_dram_pct_of_peak": heavy[2] if heavy else None,
            "lsu_sector_efficiency": eff("advance_sweep"),
            "heaviest_launch": {"dram_bytes": heavy[0], "ms": heavy[1] / 1e6,
                                "GBps": heavy[0] / heavy[1] if heavy and heavy[1] else None} if heavy else None}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None)
