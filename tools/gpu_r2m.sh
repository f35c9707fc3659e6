mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "k2_schedules or bench_shape or detections or depth_maps or step or ragged" > gpurun_out/t_s1.log 2>&1; tail -3 gpurun_out/t_s1.log
bash tools/gpu_sweep.sh "FD_TAIL_N=8" "FD_TAIL_N=8" 2>&1 | grep -v "^  \|Trace\|json\|raise\|obj, end" | tee gpurun_out/sweep_r2m.txt
