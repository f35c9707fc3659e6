# full round check on one B200: gpu tests, smoke, bench, ncu launch list, ncu --set full
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 400 python bench.py --steps 5 --warmup 3 > gpurun_out/b.json 2>gpurun_out/b.err; tail -3 gpurun_out/b.err
python -c "import json;d=json.load(open('gpurun_out/b.json'));print(d['value'],d['e2e']['value'],d['roofline']['kernel'],d['roofline']['frac'],d['roofline_k2_other']['frac'],d['kernel_ms_per_step'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv \
  python bench.py --frames 64 --steps 2 --warmup 1 --no-cpu --no-e2e > gpurun_out/ncu_l.log 2>&1; tail -2 gpurun_out/ncu_l.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_stage1|k_deep1|k_tail|k_marg|k_carry|k_corner|k_tile|k_group" -c 8 -o gpurun_out/full_r1c -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
