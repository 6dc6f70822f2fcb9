#!/usr/bin/env python
"""Per-CUDA-source-line instruction counts and stall samples of a --set full --import-source capture:
    python tools/ncu_lines.py <prof.ncu-rep> [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
fname = "?"
agg = []
hdr = None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].rsplit("/", 1)[-1]
        continue
    if r[0] == "Line No":
        hdr = {h: i for i, h in enumerate(r) if h not in ("Source",)}
        hdr["Instructions Executed"] = r.index("Instructions Executed")
        hdr["Warp Stall Sampling (All Samples)"] = r.index("Warp Stall Sampling (All Samples)")
        continue
    if hdr is None or not r[0]:
        continue
    try:
        ins = float(r[hdr["Instructions Executed"]])
        smp = float(r[hdr["Warp Stall Sampling (All Samples)"]])
    except (ValueError, IndexError):
        continue
    agg.append((ins, smp, f"{fname}:{r[0]}", r[1].strip()[:100]))
ti = sum(a[0] for a in agg)
ts = sum(a[1] for a in agg)
agg.sort(key=lambda x: -x[0])
print(f"total warp instructions {ti:.4g}, stall samples {ts:.0f}")
for ins, smp, loc, src in agg[:top]:
    print(f"{100 * ins / ti:5.1f}% ins {100 * smp / max(ts, 1):5.1f}% smp  {loc:22s} {src}")
