"""k_deepq bring-up: one small detect (c2 frames) against the oracle; prints the outcome."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import fdgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
W, H, s = 640, 480, 1.2
text = open(os.path.join(ROOT, "cascades", "c2.fdc")).read()
lv = oracle.plan(W, H, 24, s, 1)
fr, _ = fdgen.frames(2, 5, 3, W, H, lv, faces="fixed", face_param=3, max_face_level=12)
casc = fd.Cascade(text)
got = fd.to_numpy(fd.fd_detect(casc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 20))
torch.cuda.synchronize()
ref, _ = oracle.detect(oracle.Cascade(text), fr, 24, s, 1, nthreads=os.cpu_count())
print("detections", len(got), len(ref), "equal", np.array_equal(got, ref))
