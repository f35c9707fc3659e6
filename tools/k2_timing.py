#!/usr/bin/env python3
"""Diagnostic: K2 phase cycles per tile (needs libfd_timing.so, FD_LIB_VARIANT=timing)."""
import ctypes as C
import os
import sys

os.environ.setdefault("FD_LIB_VARIANT", "timing")
os.environ.setdefault("FD_JIT", "0")   # the phase counters live in the generic K2
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import fdgen  # noqa: E402
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

L = fd.lib()
L.fd_debug_k2_timing.argtypes = [C.c_void_p, C.c_int]
W, H, s = 1920, 1080, 1.1
plan = fd.fd_pyramid_plan(W, H, 24, s, 1)
fr, _ = fdgen.frames(4, 0, 32, W, H, [(f, w, h) for (f, w, h, _) in plan], faces="poisson", face_param=4,
                     max_face_level=30)
casc = fd.Cascade.from_file(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "cascades", "c3.fdc"))
d = torch.from_numpy(fr).cuda()
fd.fd_detect(casc, d, 24, s, 1, capacity=1 << 20)
buf = (C.c_ulonglong * 128)()
L.fd_debug_k2_timing(buf, 1)
fd.fd_detect(casc, d, 24, s, 1, capacity=1 << 20)
torch.cuda.synchronize()
L.fd_debug_k2_timing(buf, 0)
t = buf[0]
print(f"tiles {t}  per tile cycles: tma-wait {buf[1]/t:.0f}  stage1 {buf[2]/t:.0f}  deep {buf[3]/t:.0f}")
print("tiles by deep-loop exit stage:", [buf[4 + i] for i in range(12)])
print(f"tail: {buf[81]} warps, {buf[80]/max(buf[81],1):.0f} cycles each; mode M {buf[82]/t:.0f} / mode L {buf[83]/t:.0f} cycles per tile")
for i in range(1, 32):
    if buf[48 + i]:
        print(f"  stage {i:2d}: {buf[48+i]:8d} tiles  {buf[16+i]/buf[48+i]:8.0f} cycles/tile  {buf[16+i]/t:8.0f} per tile overall")
