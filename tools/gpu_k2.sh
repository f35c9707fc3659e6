# quick K2 check: parity subset + truncation timings + bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
MODE=detect timeout 300 python tools/k2_truncate.py r1:10 25
for v in "$@"; do
  env $v timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/sw.json 2>gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$v', round(d['value'],1), {a:round(b,2) for a,b in k.items()})" || tail -5 gpurun_out/sw.err
done
