"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 14 and r[0] != "ID"]
agg = defaultdict(lambda: [0, 0.0])
for r in rows:
    name = r[4].split("(")[0]
    name = name[:90]
    agg[name][0] += 1
    agg[name][1] += float(r[14]) / 1e6
tot = sum(v[1] for v in agg.values())
print(f"{'kernel':92s} {'launches':>8s} {'total_ms':>10s} {'share':>7s}")
for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:92s} {n:8d} {t:10.3f} {100 * t / tot:6.2f}%")
print(f"{'TOTAL':92s} {sum(v[0] for v in agg.values()):8d} {tot:10.3f}")
