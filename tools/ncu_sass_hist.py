"""Aggregate an `ncu --page source --csv --print-source=sass` export: executed warp-instructions
and stall samples per opcode, and the hottest address ranges."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
data = rows[2:]
op_inst = defaultdict(float)
op_samp = defaultdict(float)
tot_i = tot_s = 0.0
seq = []
for r in data:
    if len(r) < len(hdr):
        continue
    src = r[ix["Source"]].strip()
    op = src.split()[0] if src else "?"
    if op.startswith("@"):
        op = src.split()[1]
    ie = float(r[ix["Instructions Executed"]] or 0)
    sm = float(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    op_inst[op] += ie
    op_samp[op] += sm
    tot_i += ie
    tot_s += sm
    seq.append((r[ix["Address"]], src, ie, sm))
print(f"total warp-instructions {tot_i:.3e}, stall samples {tot_s:.0f}")
for op, v in sorted(op_inst.items(), key=lambda t: -t[1])[:25]:
    print(f"  {op:28s} inst {v / tot_i * 100:5.1f}%  samples {op_samp[op] / max(tot_s, 1) * 100:5.1f}%")
# hottest windows of 16 consecutive instructions by samples
w = 24
best = sorted(range(0, max(1, len(seq) - w)), key=lambda i: -sum(s[3] for s in seq[i:i + w]))
shown = []
for i in best:
    if any(abs(i - j) < w for j in shown):
        continue
    shown.append(i)
    if len(shown) > int(sys.argv[2] if len(sys.argv) > 2 else 6):
        break
    ss = sum(s[3] for s in seq[i:i + w])
    ii = sum(s[2] for s in seq[i:i + w])
    print(f"--- {seq[i][0]}: samples {ss / tot_s * 100:.1f}%, inst {ii / tot_i * 100:.1f}%")
    for a, src, ie, sm in seq[i:i + w]:
        print(f"   {a} {ie:12.0f} {sm:7.0f}  {src[:90]}")
