"""Soft-cascade test inputs (row f4, reading R8b) derived from the committed synthetic cascades.

A pure text transformation of a .fdc file -- no detection arithmetic: the stumps are kept in
order and each stage threshold becomes a threshold on the running sum, the sum of the hard
thresholds so far (so pass rates stay in the range the hard cascade was calibrated for).
per_stump=True splits every stage into one-stump stages, the per-stump rejection trace of a
Bourdev-Brandt soft cascade; the threshold after stump j of stage s (n_s stumps) is
acc_{s-1} + (j+1)/n_s * T_s, written as the nearest float32."""
import os

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _f(tok):
    return float.fromhex(tok) if "0x" in tok else float(tok)


def soft_from(name, n_stages=None, per_stump=False):
    lines = open(os.path.join(ROOT, "cascades", name)).read().splitlines()
    head, stages = [], []
    for ln in lines:
        t = ln.split()
        if not t or t[0].startswith("#") or t[0] in ("FDC", "window", "stages"):
            continue
        if t[0] == "filter":
            head.append(ln)
        elif t[0] == "stage":
            stages.append((_f(t[2]), []))
        elif t[0] == "stump":
            stages[-1][1].append(ln)
    if n_stages is not None:
        stages = stages[:n_stages]
    body, acc, count = [], 0.0, 0
    for T, stumps in stages:
        if per_stump:
            for j, sl in enumerate(stumps):
                body += [f"stage 1 {np.float32(acc + (j + 1) / len(stumps) * T).item()!r}", sl]
                count += 1
        else:
            body += [f"stage {len(stumps)} {np.float32(acc + T).item()!r}"] + stumps
            count += 1
        acc += T
    return "\n".join(["FDC 1", "window 24 24"] + head + ["soft", f"stages {count}"] + body) + "\n"
