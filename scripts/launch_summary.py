"""Per-kernel summary of an ncu --metrics gpu__time_duration.sum launch list."""
import collections, csv, sys
rows = list(csv.reader(open(sys.argv[1])))
h = None
agg = collections.defaultdict(list)
for r in rows:
    if 'Kernel Name' in r:
        h = r
        continue
    if h and len(r) == len(h) and r[h.index('Metric Name')] == 'gpu__time_duration.sum':
        agg[r[h.index('Kernel Name')][:70]].append(float(r[h.index('Metric Value')]))
tot = sum(sum(v) for v in agg.values())
print(f"{'launches':>8} {'avg us':>10} {'share':>7}  kernel")
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{len(v):8d} {sum(v) / len(v) / 1000:10.2f} {100 * sum(v) / tot:6.1f}%  {k}")
