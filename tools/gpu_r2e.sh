mkdir -p gpurun_out
FD_S_TAIL=2 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_f1|k_tail" -c 2 -o gpurun_out/f1_st2 -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_st2.log 2>&1; tail -2 gpurun_out/ncu_st2.log
