# ncu --set full of one K2 launch (16 1080p frames), JIT and generic builds
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_stage1|k_deep1" -c 2 -o gpurun_out/k2_jit -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_jit.log 2>&1
FD_JIT=0 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_stage1|k_deep1" -c 2 -o gpurun_out/k2_gen -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_gen.log 2>&1
tail -2 gpurun_out/ncu_jit.log gpurun_out/ncu_gen.log
