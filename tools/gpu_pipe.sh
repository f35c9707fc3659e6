# pipeline A/B + gpu tests + ncu full capture of the K2/K1 kernels (16 frames)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
for P in 0 1; do
  FD_PIPE=$P timeout 400 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/b_pipe$P.json 2>gpurun_out/b_pipe$P.err; tail -2 gpurun_out/b_pipe$P.err
  python -c "import json;d=json.load(open('gpurun_out/b_pipe$P.json'));print('pipe$P',d['value'],d['e2e']['value'],d['roofline']['kernel'],d['roofline']['frac'],d['roofline_k2_other']['frac'],{k:round(v,1) for k,v in d['kernel_ms_per_step'].items()})"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_stage1|k_deep1|k_tail|k_marg|k_carry|k_corner|k_tile|k_group" -c 8 -o gpurun_out/full_r1b -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
