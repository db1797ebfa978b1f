#!/usr/bin/env python
"""Top source lines of a kernel in an ncu report: warp-stall samples and
instructions executed per CUDA source line (needs -lineinfo + --import-source).
usage: ncu_lines.py <report.ncu-rep> [top=25]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, fname, hdr = [], None, None
for r in csv.reader(io.StringIO(raw)):
    if not r:
        continue
    if r[0] in ("File Path", "File Name"):
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr[:2], r[:2]))
        d.update(zip(hdr[4:], r[4:]))
        try:
            s = float(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
            ins = float(d.get("Instructions Executed", "0") or 0)
        except ValueError:
            continue
        if (s or ins) and d["Line No"].strip():
            rows.append((s, ins, fname, d["Line No"], d["Source"][:110]))
agg = {}
for s, ins, f, ln, src in rows:
    k = (f, ln)
    a = agg.setdefault(k, [0.0, 0.0, src])
    a[0] += s
    a[1] += ins
rows = [(v[0], v[1], k[0], k[1], v[2]) for k, v in agg.items()]
tot_s = sum(r[0] for r in rows) or 1
tot_i = sum(r[1] for r in rows) or 1
print(f"total stall samples {tot_s:.0f}, warp instructions {tot_i:.3e}")
key = 1 if "--by-inst" in sys.argv else 0
for s, ins, f, ln, src in sorted(rows, key=lambda r: -r[key])[:top]:
    print(f"{s / tot_s:6.1%} {ins / tot_i:6.1%}  {f}:{ln:5s} {src}")
