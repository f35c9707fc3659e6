#!/usr/bin/env python3
"""Per-source-line summary of an ncu report (--page source, cuda view): warp-stall samples,
instructions, shared-memory wavefronts and top stall reasons.  Usage: ncu_lines.py rep [top]"""
import csv
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, f, hdr = [], None, None
for r in csv.reader(out.splitlines()):
    if not r:
        continue
    if r[0] == "File Path" or r[0] == "File Name":
        f = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r[0].isdigit():
        continue
    d = dict(zip(hdr, r))
    d["_file"] = f
    rows.append(d)


def num(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


tot = sum(num(d.get("Warp Stall Sampling (All Samples)", 0)) for d in rows)
stalls = [h for h in (hdr or []) if h.startswith("stall_") and "Not Issued" not in h]
rows.sort(key=lambda d: -num(d.get("Warp Stall Sampling (All Samples)", 0)))
print(f"total samples {tot:.0f}")
print(f"{'file:line':28s} {'samp%':>6s} {'inst':>10s} {'smemWF':>10s} {'excess':>9s}  top stalls / source")
for d in rows[:top]:
    s = num(d.get("Warp Stall Sampling (All Samples)", 0))
    st = sorted(((num(d.get(h, 0)), h[6:]) for h in stalls), reverse=True)[:3]
    sts = " ".join(f"{n}:{v/max(s,1)*100:.0f}%" for v, n in st if v > 0)
    print(f"{d['_file'] + ':' + d['Line No']:28s} {s/tot*100:6.2f} {num(d.get('Instructions Executed',0)):10.0f} "
          f"{num(d.get('L1 Wavefronts Shared',0)):10.0f} {num(d.get('L1 Wavefronts Shared Excessive',0)):9.0f}  {sts}  | {d['Source'][:70]}")
