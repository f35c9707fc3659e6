mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "c6q or packed16 or c6_workload" > gpurun_out/t_f3.log 2>&1; tail -3 gpurun_out/t_f3.log
for c in c6 c6q; do
  timeout 400 python bench.py --cascade $c --steps 3 --warmup 2 --no-cpu --no-e2e > gpurun_out/b_$c.json 2>gpurun_out/b_$c.err; tail -2 gpurun_out/b_$c.err
  python -c "import json;d=json.load(open('gpurun_out/b_$c.json'));print('$c', round(d['value'],1), {a: round(b, 2) for a, b in d['kernel_ms_per_step_one_slot'].items()})"
done
