mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "integral or pyramid or depth_maps_bit_exact or filter or min_size or ragged or k2_schedules" > gpurun_out/t_k1.log 2>&1; tail -3 gpurun_out/t_k1.log
bash tools/gpu_sweep.sh "FD_TAIL_N=8" "FD_TAIL_N=4" 2>&1 | grep -v "^  \|Trace\|json\|raise\|obj, end" | tee gpurun_out/sweep_r2k.txt
