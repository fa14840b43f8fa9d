"""Stall samples aggregated per CUDA source line of an .ncu-rep (needs -lineinfo builds).
Usage: python tools/ncu_src.py <file.ncu-rep> [ntop]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr_i = next(i for i, r in enumerate(rows) if "Warp Stall Sampling (All Samples)" in r)
h = rows[hdr_i]
i_s = h.index("Warp Stall Sampling (All Samples)")
i_src = h.index("Source") if "Source" in h else 1
i_ln = h.index("Line") if "Line" in h else 0
data = [r for r in rows[hdr_i + 1:] if len(r) > i_s]
tot = sum(float(r[i_s] or 0) for r in data) or 1
for r in sorted(data, key=lambda r: -float(r[i_s] or 0))[:ntop]:
    print(f"{100 * float(r[i_s]) / tot:5.1f}%  L{r[i_ln]:>5}  {r[i_src].strip()[:110]}")
