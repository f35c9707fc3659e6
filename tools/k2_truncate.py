#!/usr/bin/env python3
"""Diagnostic: K2 time per 1080p frame with the c3 cascade truncated to its first k stages
(how much each deeper stage adds on top of the dense first stage)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import fdgen  # noqa: E402
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
W, H, s, F = 1920, 1080, 1.1, int(os.environ.get("FRAMES", "32"))
text = open(os.path.join(ROOT, "cascades", "c3.fdc")).read().split("\n")
hdr, stages, cur = [], [], None
for ln in text:
    t = ln.split()
    if t and t[0] == "stage":
        cur = [ln]
        stages.append(cur)
    elif t and t[0] == "stump":
        cur.append(ln)
    elif t and t[0] not in ("stages",):
        hdr.append(ln)
plan = fd.fd_pyramid_plan(W, H, 24, s, 1)
fr, _ = fdgen.frames(4, 0, F, W, H, [(f, w, h) for (f, w, h, _) in plan], faces="poisson", face_param=4,
                     max_face_level=30)
d = torch.from_numpy(fr).cuda()
for arg in sys.argv[1:] or ["1", "2", "3", "4", "6", "10", "25"]:
    if arg.startswith("r1:"):      # first stage cut to j stumps, threshold that rejects every window
        k, j = 1, int(arg[3:])
        sts = [[f"stage {j} 1e30"] + stages[0][1:1 + j]]
    elif arg.startswith("s1:"):    # first stage cut to j stumps (threshold kept)
        k, j = 1, int(arg[3:])
        t0 = stages[0][0].split()
        sts = [[f"stage {j} {t0[2]}"] + stages[0][1:1 + j]]
    else:
        k = int(arg)
        sts = stages[:k]
    body = "\n".join(h for h in hdr if h.strip()) + f"\nstages {k}\n" + "\n".join("\n".join(st) for st in sts) + "\n"
    casc = fd.Cascade(body)
    run = (lambda: fd.fd_detect(casc, d, 24, s, 1, capacity=1 << 26)) if os.environ.get("MODE") == "detect" else \
        (lambda: fd.fd_detect_depth(casc, d, 24, s, 1))
    run()
    torch.cuda.synchronize()
    fd.fd_profile_reset(True)
    for _ in range(3):
        run()
    torch.cuda.synchronize()
    p = fd.fd_profile_read()
    us = {k: p[k][1] / 3 / F * 1000 for k in ("cascade", "deep", "tail") if k in p and p[k][0]}
    print(f"{arg:>5s}: K2 {sum(us.values()):.1f} us/frame  " + "  ".join(f"{k} {v:.1f}" for k, v in us.items()))
