mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "k2_schedules or bench_shape or worked or small" > gpurun_out/t_sched.log 2>&1; tail -5 gpurun_out/t_sched.log
bash tools/gpu_sweep.sh "FD_TAIL_N=8" "FD_S_TAIL=2" "FD_S_TAIL=3" "FD_S_TAIL=4" "FD_S_TAIL=5" "FD_S_TAIL=3 FD_TAIL_SMEM_STUMPS=0" "FD_S_TAIL=3 FD_F1_GROUP_MB=32" 2>&1 | tee gpurun_out/sweep_r2d.txt
