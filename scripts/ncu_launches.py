"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list: per-kernel totals and shares,
plus the launches of the last N kernels (one BFS)."""
import collections
import csv
import sys


def load(path):
    lines = open(path).read().splitlines()
    start = [i for i, l in enumerate(lines) if l.startswith('"ID"')][0]
    rows = list(csv.reader(lines[start:]))
    hdr = rows[0]
    ki, vi, ii = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("ID")
    return [(int(r[ii]), r[ki].split("(")[0], float(r[vi].replace(",", ""))) for r in rows[1:] if len(r) > vi and r[vi]]


if __name__ == "__main__":
    data = load(sys.argv[1])
    tail = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    for x in data[-tail:]:
        print(f"{x[0]:6d} {x[2] / 1e3:10.1f} us  {x[1]}")
    agg = collections.defaultdict(float)
    for _, k, v in data[-tail:]:
        agg[k] += v
    tot = sum(agg.values())
    print(f"--- last {tail} launches: {tot / 1e3:.1f} us")
    for k, v in sorted(agg.items(), key=lambda x: -x[1]):
        print(f"{v / 1e3:10.1f} us {100 * v / tot:5.1f}%  {k}")
