"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per-kernel count, total, share."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if r and r[0] == 'ID')
hdr, data = rows[start], rows[start + 1:]
k, v = hdr.index('Kernel Name'), hdr.index('Metric Value')
agg = collections.defaultdict(list)
for r in data:
    agg[r[k].split('(')[0]].append(float(r[v].replace(',', '')))
tot = sum(sum(x) for x in agg.values())
print(f"{'launches':>8} {'total ms':>10} {'share':>6} {'mean us':>10}  kernel (ncu --metrics gpu__time_duration.sum, "
      f"--clock-control none; cold-cache, serialised)")
for name, xs in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{len(xs):8d} {sum(xs) / 1e6:10.3f} {sum(xs) / tot * 100:5.1f}% {sum(xs) / len(xs) / 1e3:10.1f}  {name}")
