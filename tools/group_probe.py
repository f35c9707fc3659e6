#!/usr/bin/env python3
"""Diagnostic: fd_group alone on the detections of N c4 frames (for ncu launch lists)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import fdgen  # noqa: E402
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
W, H, s, F = 1920, 1080, 1.1, int(os.environ.get("FRAMES", "128"))
plan = fd.fd_pyramid_plan(W, H, 24, s, 1)
fr, _ = fdgen.frames(4, 0, F, W, H, [(f, w, h) for (f, w, h, _) in plan], faces="poisson", face_param=4,
                     max_face_level=30)
casc = fd.Cascade.from_file(os.path.join(ROOT, "cascades", "c3.fdc"))
d = torch.from_numpy(fr).cuda()
dets = fd.fd_detect(casc, d, 24, s, 1, capacity=1 << 22)
torch.cuda.synchronize()
for _ in range(3):
    g = fd.fd_group(dets, 0.5, 1)
torch.cuda.synchronize()
fd.fd_profile_reset(True)
g = fd.fd_group(dets, 0.5, 1)
torch.cuda.synchronize()
print(dets.shape[0], g.shape[0], fd.fd_profile_read()["group"])
import numpy as np  # noqa: E402
fcount = np.bincount(fd.to_numpy(dets)["frame"], minlength=F)
print("detections per frame: max", fcount.max(), "p99", np.percentile(fcount, 99), "mean", fcount.mean(),
      "top", sorted(fcount)[-5:])
if os.environ.get("SPLIT"):      # time fd_group per frame for the 5 largest frames
    d_np = fd.to_numpy(dets)
    for f in np.argsort(fcount)[-5:]:
        sub = dets[torch.from_numpy(d_np["frame"] == f).cuda()]
        fd.fd_group(sub, 0.5, 1)
        torch.cuda.synchronize()
        fd.fd_profile_reset(True)
        fd.fd_group(sub, 0.5, 1)
        torch.cuda.synchronize()
        print("frame", f, fcount[f], fd.fd_profile_read()["group"])
