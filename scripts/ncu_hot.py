"""Per-SASS-instruction hot spots of an ncu report (instructions executed, stall samples)."""
import csv, io, subprocess, sys
path = sys.argv[1]
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.004
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
tot = sum(d[2] for d in data)
totsm = sum(d[3] for d in data)
print("total warp-instructions", tot, "stall samples", totsm)
for a, s, e, sm in data:
    if e > tot * thr or sm > totsm * thr * 1.5:
        print(f"{a[-5:]} {e / tot * 100:6.2f}% {sm / totsm * 100:6.2f}%  {s}")
