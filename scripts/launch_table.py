"""Per-launch table from an ncu --csv launch list with time + dram bytes metrics.

    python scripts/launch_table.py gpurun_out/X.csv [skip_first_n]"""
import collections
import csv
import sys

lines = open(sys.argv[1]).read().splitlines()
start = [i for i, l in enumerate(lines) if l.startswith('"ID"')][0]
rows = list(csv.reader(lines[start:]))
hdr = rows[0]
ki, mi, vi, ii = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
L = collections.OrderedDict()
for r in rows[1:]:
    if len(r) <= vi:
        continue
    k = int(r[ii])
    L.setdefault(k, {"name": r[ki].split("(")[0].replace("void ", "").replace("sg::", "")})
    L[k][r[mi]] = float(r[vi].replace(",", ""))
skip = int(sys.argv[2]) if len(sys.argv) > 2 else 0
agg = collections.defaultdict(lambda: [0.0, 0.0, 0])
tot_t = 0
for k, d in list(L.items())[skip:]:
    t = d.get("gpu__time_duration.sum", 0) / 1e3
    b = (d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0))
    print(f"{k:5d} {t:9.1f} us {b / 1e6:9.1f} MB {b / (t * 1e3) if t else 0:8.0f} GB/s  {d['name']}")
    agg[d["name"]][0] += t
    agg[d["name"]][1] += b
    agg[d["name"]][2] += 1
    tot_t += t
print(f"--- total {tot_t:.1f} us")
for n, (t, b, c) in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{t:9.1f} us {100 * t / tot_t:5.1f}% {c:4d} launches {b / 1e6:9.1f} MB  {n}")
