# launch list + ncu --set full of the default path (one launch of each kernel), summaries under gpurun_out/
mkdir -p gpurun_out
TAG=${TAG:-r2}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --frames 64 --steps 2 --warmup 1 --no-cpu --no-e2e > gpurun_out/ncu_l.log 2>&1; tail -2 gpurun_out/ncu_l.log
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"${KRE:-k_stage1|k_deep1|k_tail|k_marg|k_carry|k_corner|k_tile|k_group|k_f1|k_level}" -c ${NK:-12} -o gpurun_out/full_$TAG -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
