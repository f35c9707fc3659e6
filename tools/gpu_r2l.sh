mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_marg|k_tile" -c 2 -o gpurun_out/k1_r2 -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_k1.log 2>&1; tail -2 gpurun_out/ncu_k1.log
