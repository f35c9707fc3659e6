mkdir -p gpurun_out
bash tools/gpu_sweep.sh "FD_TAIL_N=8" "FD_TAIL_N=32" "FD_TAIL_N=128" "FD_TAIL_N=8 FD_F1_GROUP_MB=256" "FD_TAIL_N=8 FD_LANE_MIN=8" "FD_F1=0" 2>&1 | tee gpurun_out/sweep_r2c.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_f1|k_tail|k_level" -c 3 -o gpurun_out/f1_full -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
