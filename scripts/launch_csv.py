"""Print per-launch kernel times (µs) from an ncu --csv launch list: python scripts/launch_csv.py FILE [FILE2]"""
import csv
import sys


def load(p):
    rows = [r for r in csv.DictReader(l for l in open(p) if l.startswith('"'))]
    return [(r['Kernel Name'].split('(')[0].replace('void ', '').replace('sg::', ''), float(r['Metric Value']) / 1000)
            for r in rows if r['Metric Name'] == 'gpu__time_duration.sum']


a = load(sys.argv[1])
b = load(sys.argv[2]) if len(sys.argv) > 2 else []
for i in range(max(len(a), len(b))):
    x = f"{a[i][0]:28s} {a[i][1]:8.1f}" if i < len(a) else " " * 37
    y = f"   {b[i][0]:28s} {b[i][1]:8.1f}" if i < len(b) else ""
    print(f"{i:4d} {x}{y}")
