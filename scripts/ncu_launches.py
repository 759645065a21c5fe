"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per-kernel count, time
and share of the match step.  Only the launches of the last K match calls are counted (a call
starts with k_hash_vocab; the build and the warm-up/tuning calls before them are dropped), and
torch's own kernels (the L2 flush between steps) are left out.
usage: ncu_launches.py <launches.csv> [K=2]"""
import collections, csv, sys
rows = list(csv.reader(open(sys.argv[1])))
K = int(sys.argv[2]) if len(sys.argv) > 2 else 2
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[start]
iname, ival = hdr.index("Kernel Name"), hdr.index("Metric Value")
launches = [r for r in rows[start + 1:] if len(r) > ival]
calls = [i for i, r in enumerate(launches) if "k_hash_vocab" in r[iname]]
first = calls[-K] if len(calls) >= K else 0
agg = collections.defaultdict(lambda: [0, 0.0])
for r in launches[first:]:
    if "at::" in r[iname] or "at_cuda" in r[iname]:
        continue
    n = r[iname].split("(")[0][-60:]
    agg[n][0] += 1
    agg[n][1] += float(r[ival].replace(",", ""))
tot = sum(v[1] for v in agg.values())
print(f"last {K} match calls ({len(launches) - first} launches of {len(launches)})")
print(f"{'launches':>8} {'total ms':>10} {'share':>6}  kernel   (cold-cache, serialised ncu times; compare shares)")
for n, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{c:8d} {v / 1e6:10.3f} {100 * v / tot:5.1f}%  {n}")
