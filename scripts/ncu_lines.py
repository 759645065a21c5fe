"""Warp-instructions and stall samples of the hot kernel per CUDA source line (ncu source page,
cuda,sass view).  usage: ncu_lines.py <rep> [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["/usr/local/cuda/bin/ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
hdr = rows[hi]
iex = hdr.index("Instructions Executed")
ism = hdr.index("Warp Stall Sampling (All Samples)")
lines = []
for r in rows[hi + 1:]:
    if r and r[0] and r[0] != "Line No":
        try:
            lines.append((int(r[0]), r[1].strip()[:90], int(r[iex]), int(r[ism])))
        except ValueError:
            pass
tot = sum(l[2] for l in lines) or 1
tsm = sum(l[3] for l in lines) or 1
print(f"total warp-instructions {tot}")
for ln, src, ex, sm in sorted(lines, key=lambda l: -l[2])[:top]:
    print(f"{ln:5d} {ex / tot * 100:5.1f}% stall {sm / tsm * 100:5.1f}%  {src}")
