#!/usr/bin/env python3
"""Write the compressed f3 workload cascade ("reencoding and combining
them into two 16-bit words"): cascades/c6q.fdc = the OpenCV-shaped c6 cascade with every stump's
theta / left / right rounded to IEEE binary16 (round to nearest even) and the line
'compress packed16', so the oracle and the library evaluate the stumps decoded from the compressed
words (reading R13).  Stage thresholds stay binary32.  Input generation only: calls no product code;
the oracle checks that every value is exactly representable when it parses the file."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def f16(v: str) -> str:
    x = float.fromhex(v) if "x" in v else float(v)
    return float(np.float32(np.float16(x))).hex()


def main(src="c6.fdc", dst="c6q.fdc"):
    out = []
    for line in open(os.path.join(ROOT, "cascades", src)):
        t = line.split()
        if t and t[0] == "window":
            out.append(line.rstrip("\n"))
            out.append("compress packed16")
            continue
        if t and t[0] == "stump":
            nr = int(t[1])
            b = 2 + 5 * nr
            t[b:b + 3] = [f16(v) for v in t[b:b + 3]]
            out.append(" ".join(t))
            continue
        if t and t[0].startswith("#"):
            out.append(f"# {dst}: {src} with binary16 theta/left/right, compressed records (tools/make_packed_cascade.py)")
            continue
        out.append(line.rstrip("\n"))
    with open(os.path.join(ROOT, "cascades", dst), "w") as fh:
        fh.write("\n".join(out) + "\n")


if __name__ == "__main__":
    main(*sys.argv[1:])
