"""Group SASS instructions of an ncu report into runs of equal execution count (basic blocks)."""
import csv, io, subprocess, sys
path = sys.argv[1]
out = subprocess.run(["/usr/local/cuda/bin/ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ia, isrc, iex, ism = (hdr.index(k) for k in ("Address", "Source", "Instructions Executed", "Warp Stall Sampling (All Samples)"))
data = []
for r in rows[2:]:
    try:
        data.append((r[ia], r[isrc].strip(), int(r[iex]), int(r[ism])))
    except Exception:
        pass
tot = sum(d[2] for d in data); totsm = sum(d[3] for d in data)
blocks = []
for a, s, e, sm in data:
    if blocks and blocks[-1]["e"] == e:
        b = blocks[-1]; b["n"] += 1; b["sm"] += sm; b["last"] = a; b["src"].append(s)
    else:
        blocks.append({"first": a, "last": a, "e": e, "n": 1, "sm": sm, "src": [s]})
for b in blocks:
    share = b["e"] * b["n"] / tot
    if share > 0.01 or b["sm"] / totsm > 0.01:
        print(f"{b['first'][-5:]}-{b['last'][-5:]} n={b['n']:3d} exec/inst={b['e']:>11d} inst%={100*share:5.1f} stall%={100*b['sm']/totsm:5.1f}  {b['src'][0][:40]} .. {b['src'][-1][:40]}")
