mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_deepq" -c 1 -o gpurun_out/dq_full -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_dq.log 2>&1; tail -3 gpurun_out/ncu_dq.log
