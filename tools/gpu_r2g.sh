mkdir -p gpurun_out
for cfg in "FD_PIPE=0" "FD_PIPE=0 FD_DEEP_SPLIT=0" "FD_PIPE=0 FD_S_TAIL=2" "FD_PIPE=0 FD_TAIL_N=32"; do
  echo "== $cfg"; env $cfg timeout 300 python tools/k2_timing.py 2>&1 | tail -32
done > gpurun_out/timing_r2g.txt
cat gpurun_out/timing_r2g.txt
