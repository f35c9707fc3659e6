# quick A/B: gpu parity tests (fast subset) + bench with FD_PIPE=0 and 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q ${FD_TESTS:-} > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
for P in 0 1; do
  FD_PIPE=$P timeout 400 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/b_pipe$P.json 2>gpurun_out/b_pipe$P.err; tail -2 gpurun_out/b_pipe$P.err
  python -c "import json;d=json.load(open('gpurun_out/b_pipe$P.json'));print('pipe$P',round(d['value'],1),d['roofline']['kernel'],round(d['roofline']['frac'],3),round(d['roofline_k2_other']['frac'],3),{k:round(v,1) for k,v in d['kernel_ms_per_step'].items()})"
done
