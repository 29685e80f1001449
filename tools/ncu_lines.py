#!/usr/bin/env python
"""Per-source-line instruction counts and stall samples of one kernel in an ncu report
(`ncu -i REP --page source --csv --print-source cuda,sass`), hottest lines first.

    python tools/ncu_lines.py gpurun_out/x.ncu-rep [top]
"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
fname = ""
rows = []
hdr = None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr and r[0] and r[0] != "Function Name":
        d = dict(zip(hdr[2:], r[2:]))
        try:
            rows.append((int(d["Instructions Executed"]), int(d["Warp Stall Sampling (All Samples)"]), fname, r[0], r[1]))
        except (KeyError, ValueError):
            pass
tot_i = sum(x[0] for x in rows) or 1
tot_s = sum(x[1] for x in rows) or 1
print(f"total warp instructions {tot_i:.3e}, samples {tot_s}")
for ins, smp, f, ln, src in sorted(rows, key=lambda x: -x[0])[:top]:
    print(f"{100*ins/tot_i:5.1f}% inst {100*smp/tot_s:5.1f}% stall  {f}:{ln}  {src.strip()[:90]}")
