"""compute-sanitizer workload: one small call of every kernel family on cuda:0 (c1 and c2 frames,
default schedule and, with FD_F1=1 in the environment, the f1 schedule): fd_detect_depth,
fd_detect (+ stage counters), fd_group, fd_integral, fd_build_pyramid, fd_depth_histogram."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import fdgen  # noqa: E402
import oracle  # noqa: E402  (only for the pyramid plan used to plant faces)
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
for cfg, (W, H, s) in ((1, (320, 240, 1.25)), (2, (640, 480, 1.2))):
    casc = fd.Cascade.from_file(os.path.join(ROOT, "cascades", f"c{cfg}.fdc"))
    lv = oracle.plan(W, H, 24, s, 1)
    fr, _ = fdgen.frames(cfg, 0, 2, W, H, lv, faces="fixed", face_param=3, max_face_level=8)
    d = torch.from_numpy(fr).cuda()
    depth, score = fd.fd_detect_depth(casc, d, 24, s, 1)
    sc = torch.zeros(casc.n_stages + 1, dtype=torch.int64, device="cuda")
    dets = fd.fd_detect(casc, d, 24, s, 1, capacity=1 << 18, stage_counts=sc)
    grp = fd.fd_group(dets, 0.5, 1)
    fd.fd_depth_histogram(depth, 2, W, H, casc.n_stages, 24, s, 1)
    ii, sq = fd.fd_integral(d)
    fd.fd_build_pyramid(d, 24, s)
    torch.cuda.synchronize()
    print(f"c{cfg}: {int(dets.shape[0])} detections, {int(grp.shape[0])} groups")
