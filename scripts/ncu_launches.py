"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per-kernel count, time, share."""
import collections, csv, sys
rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[start]
iname, ival = hdr.index("Kernel Name"), hdr.index("Metric Value")
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[start + 1:]:
    if len(r) <= ival:
        continue
    n = r[iname].split("(")[0][-60:]
    agg[n][0] += 1
    agg[n][1] += float(r[ival].replace(",", ""))
tot = sum(v[1] for v in agg.values())
print(f"{'launches':>8} {'total ms':>10} {'share':>6}  kernel   (cold-cache, serialised ncu times; compare shares)")
for n, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{c:8d} {v / 1e6:10.3f} {100 * v / tot:5.1f}%  {n}")
