mkdir -p gpurun_out
FD_PIPE=0 MODE=detect timeout 300 python tools/k2_truncate.py 1 2 3 4 5 6 8 12 25 > gpurun_out/trunc.txt 2>&1
FD_PIPE=0 timeout 300 python tools/k2_timing.py > gpurun_out/k2t.txt 2>&1
cat gpurun_out/trunc.txt gpurun_out/k2t.txt
