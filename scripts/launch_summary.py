"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per-kernel launches,
total time and share of the step.   python scripts/launch_summary.py gpurun_out/launches.csv"""
import collections
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
iK, iV = h.index("Kernel Name"), h.index("Metric Value")
agg = collections.defaultdict(list)
for r in rows[1:]:
    agg[r[iK].split("(")[0][:70]].append(float(r[iV].replace(",", "")))
tot = sum(sum(v) for v in agg.values())
print("%-70s %6s %12s %12s %7s" % ("kernel", "n", "total_ms", "mean_ms", "share"))
for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
    print("%-70s %6d %12.3f %12.4f %7.4f" % (k, len(v), sum(v) / 1e6, sum(v) / len(v) / 1e6, sum(v) / tot))
