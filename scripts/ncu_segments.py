"""Instruction share of an ncu report's SASS by straight-line segment (runs of equal execution
count): where the warp-instructions of the hot kernel go.  usage: ncu_segments.py <rep> [min%]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
out = subprocess.run(["/usr/local/cuda/bin/ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ia, isrc, iex, ism = (hdr.index(k) for k in ("Address", "Source", "Instructions Executed",
                                             "Warp Stall Sampling (All Samples)"))
data = []
for r in rows[2:]:
    try:
        data.append((int(r[ia], 16), r[isrc].strip(), int(r[iex]), int(r[ism])))
    except Exception:
        pass
tot = sum(d[2] for d in data)
totsm = sum(d[3] for d in data) or 1
base = data[0][0]
seg, cur = [], None
for a, s, e, sm in data:
    if cur and cur[2] == e:
        cur[1] = a; cur[3] += e; cur[4] += sm; cur[5] += 1; cur[6].append(s)
    else:
        if cur:
            seg.append(cur)
        cur = [a, a, e, e, sm, 1, [s]]
seg.append(cur)
print(f"total warp-instructions {tot}")
for s0, s1, e, esum, sm, n, src in seg:
    if esum > tot * thr / 100:
        ops = " ".join(x.split()[0] if not x.startswith("@") else x.split()[1] for x in src[:6])
        print(f"{s0 - base:6x}-{s1 - base:6x} n={n:3d} exec={e:10d} share={esum / tot * 100:5.1f}% "
              f"stall={sm / totsm * 100:5.1f}%  {ops}")
