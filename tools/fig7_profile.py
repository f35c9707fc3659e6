#!/usr/bin/env python3
"""Fig. 7 analytics on the c4 workload: fd_detect_depth + fd_depth_histogram
over F synthetic 1080p frames; prints the rejection rate of each stage per scale (markdown) and
the aggregate profile next to the paper's (94.52% at stage 1, ~4% at stage 2)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import fdgen  # noqa: E402
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
W, H, s, F = 1920, 1080, 1.1, int(os.environ.get("FRAMES", "32"))
plan = fd.fd_pyramid_plan(W, H, 24, s, 1)
fr, _ = fdgen.frames(4, 0, F, W, H, [(f, w, h) for (f, w, h, _) in plan], faces="poisson", face_param=4,
                     max_face_level=30)
casc = fd.Cascade.from_file(os.path.join(ROOT, "cascades", "c3.fdc"))
N = casc.n_stages
hist = torch.zeros(len(plan), N + 1, dtype=torch.int64)
for f0 in range(0, F, 8):
    d = torch.from_numpy(fr[f0:f0 + 8]).cuda()
    depth, _ = fd.fd_detect_depth(casc, d, 24, s, 1)
    hist += fd.fd_depth_histogram(depth, d.shape[0], W, H, N, 24, s, 1).cpu()
tot = hist.sum().item()
agg = hist.sum(0)
print(f"# Fig. 7 profile: {F} synthetic c4 frames (1080p, scale 1.1, cascades/c3.fdc, {N} stages)\n")
print(f"windows {tot}; rejected at stage 1: {100 * agg[0].item() / tot:.2f}% of all windows (paper 94.52%); "
      f"at stage 2: {100 * agg[1].item() / tot:.2f}% (paper ~4%); accepted: {agg[N].item()}\n")
print("| scale k | f_k | windows | rej. stage 1 | rej. stage 2 | rej. stage 3 | rej. 4+ | accepted |")
print("|---|---|---|---|---|---|---|---|")
for k, (f, w, h, n) in enumerate(plan):
    r = hist[k]
    t = r.sum().item()
    pc = [100 * r[i].item() / t for i in range(3)]
    print(f"| {k} | {f:.3f} | {t} | {pc[0]:.2f}% | {pc[1]:.2f}% | {pc[2]:.3f}% | "
          f"{100 * r[3:N].sum().item() / t:.4f}% | {r[N].item()} |")
