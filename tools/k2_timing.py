#!/usr/bin/env python3
"""Diagnostic: K2 phase cycles (needs libfd_timing.so, FD_LIB_VARIANT=timing, generic kernels)."""
import ctypes as C
import os
import sys

os.environ.setdefault("FD_LIB_VARIANT", "timing")
os.environ.setdefault("FD_JIT", "0")   # the phase counters live in the precompiled kernels
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
fd.fd_profile_reset(True)
fd.fd_detect(casc, d, 24, s, 1, capacity=1 << 20)
torch.cuda.synchronize()
print({k: round(v[1], 3) for k, v in fd.fd_profile_read().items() if v[0]})
L.fd_debug_k2_timing(buf, 0)
b = list(buf)
if b[0]:
    print(f"tiles {b[0]}  per tile cycles: tma-wait {b[1]/b[0]:.0f}  build {b[85]/b[0]:.0f}  stage1 {b[2]/b[0]:.0f}")
nbat = max(b[84], 1)
print(f"group-mode decisions {b[95]}  undecided {b[94]}  exact recomputes {b[96]}")
print(f"deep batches {b[84]}  tiles/batch {b[92]/nbat:.2f}  pool/batch {b[93]/nbat:.1f}")
print(f"per batch cycles: fill {b[90]/nbat:.0f}  tma-wait {b[91]/nbat:.0f}  deep {b[3]/nbat:.0f}")
print("batches by deep-loop exit stage:", [b[4 + i] for i in range(12)])
print(f"tail handoffs {b[81]} windows over {b[80] and 1}")
for i in range(1, 32):
    if b[48 + i]:
        print(f"  stage {i:2d}: {b[48+i]:8d} batches  {b[16+i]/b[48+i]:8.0f} cycles/batch  {b[16+i]/nbat:8.0f} per batch overall")
