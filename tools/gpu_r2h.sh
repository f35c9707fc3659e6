mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "k2_schedules or bench_shape or worked or small or soft or step or ragged or min_size" > gpurun_out/t_sched.log 2>&1; tail -5 gpurun_out/t_sched.log
bash tools/gpu_sweep.sh "FD_TAIL_N=8" "FD_DEEP_SPLIT=0" "FD_TAIL_N=4" "FD_TAIL_N=16" "FD_F1_GROUP_MB=128" "FD_F1_GROUP_MB=32" "FD_F1=0 FD_DEEP_SPLIT=0" 2>&1 | tee gpurun_out/sweep_r2h.txt
