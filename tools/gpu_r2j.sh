mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "k2_schedules" > gpurun_out/t_sched.log 2>&1; tail -3 gpurun_out/t_sched.log
bash tools/gpu_sweep.sh "FD_K2D_THREADS=128" "FD_K2D_THREADS=64" "FD_K2D_THREADS=32" "FD_K2D_THREADS=32 FD_K2D_CTAS=12" "FD_K2D_THREADS=64 FD_K2D_CTAS=6" "FD_JIT_DEEP_STUMPS=110" "FD_K2D_THREADS=32 FD_JIT_DEEP_STUMPS=110" "FD_TAIL_N=4" 2>&1 | tee gpurun_out/sweep_r2j.txt
