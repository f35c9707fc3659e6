mkdir -p gpurun_out
FD_DEEPQ=1 FD_DQ_TAIL=255 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_deepq" -c 1 -o gpurun_out/dq_lite -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_dq.log 2>&1; tail -3 gpurun_out/ncu_dq.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_stage1|k_deep1" -c 2 -o gpurun_out/s1_full -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_s1.log 2>&1; tail -3 gpurun_out/ncu_s1.log
