"""Per-CUDA-source-line totals (stall samples, instructions executed) from an ncu report.

    python scripts/ncu_lines.py report.ncu-rep [top_n]"""
import csv
import subprocess
import sys

EXTRA = ["--launch-skip", sys.argv[3], "--launch-count", "1"] if len(sys.argv) > 3 else []
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass", *EXTRA],
                     capture_output=True, text=True).stdout
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
rows = list(csv.reader(out.splitlines()))
fname, hdr, agg = None, None, {}
cur = None
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 8:
        continue
    if r[0]:   # a CUDA source line row
        cur = (fname, int(r[0]), r[1].strip()[:90])
    if r[2] and cur is not None:   # a SASS row under it
        try:
            samp = int(r[4]) if r[4] else 0
            inst = int(r[7]) if r[7] else 0
        except ValueError:
            continue
        a = agg.setdefault(cur, [0, 0])
        a[0] += samp
        a[1] += inst
tot_s = sum(v[0] for v in agg.values()) or 1
tot_i = sum(v[1] for v in agg.values()) or 1
print(f"total samples {tot_s}, warp instructions {tot_i}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{100 * v[0] / tot_s:5.1f}% smp {100 * v[1] / tot_i:5.1f}% inst  {k[0]}:{k[1]}  {k[2]}")
