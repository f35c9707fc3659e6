mkdir -p gpurun_out
timeout 300 python tools/k2_timing.py > gpurun_out/k2t.txt 2>&1
MODE=detect timeout 300 python tools/k2_truncate.py r1:10 s1:10 1 2 3 4 6 10 25 > gpurun_out/trunc.txt 2>&1
FD_JIT=0 MODE=detect timeout 300 python tools/k2_truncate.py r1:10 1 2 25 > gpurun_out/trunc_nojit.txt 2>&1
