"""Per-kernel share of an ncu launch list (--metrics gpu__time_duration.sum --csv --log-file).
usage: python scripts/launch_summary.py launches.csv"""
import collections
import csv
import sys

lines = open(sys.argv[1]).read().splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
rows = list(csv.reader(lines[start:]))
h = rows[0]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
agg = collections.defaultdict(list)
for r in rows[1:]:
    agg[r[ki][:100]].append(float(r[vi]) / 1e6)
tot = sum(sum(v) for v in agg.values())
print("ncu launch list (cold, serialised; --clock-control none): %d launches, %.3f ms" % (sum(len(v) for v in agg.values()), tot))
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print("%6.1f%%  n=%3d  mean %.4f ms  min %.4f  max %.4f  %s" % (100 * sum(v) / tot, len(v), sum(v) / len(v), min(v), max(v), k))
