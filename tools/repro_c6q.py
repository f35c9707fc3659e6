"""Debug helper: fd_detect with the compressed c6q cascade on N 1080p frames."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import fdgen  # noqa: E402
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 32
depth_first = len(sys.argv) > 2 and sys.argv[2] == "depth"
W, H, s = 1920, 1080, 1.1
plan = fd.fd_pyramid_plan(W, H, 24, s, 1)
fr, _ = fdgen.frames(4, 0, n, W, H, [(f, w, h) for (f, w, h, _) in plan], faces="poisson", face_param=4,
                     max_face_level=30)
casc = fd.Cascade.from_file(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "cascades", os.environ.get("CASC", "c6q.fdc")))
d = torch.from_numpy(fr).cuda()
if depth_first:
    fd.fd_detect_depth(casc, d[:1], 24, s, 1)
    torch.cuda.synchronize()
    print("depth ok", flush=True)
dets = fd.fd_detect(casc, d, 24, s, 1, capacity=1 << 21)
torch.cuda.synchronize()
print("detect ok", dets.shape, flush=True)
