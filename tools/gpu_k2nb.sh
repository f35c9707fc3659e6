# K2 batching check: GPU parity tests, then bench K2 ms for several tiles-per-batch settings
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
for nb in 1 2 3 4 6; do
  FD_K2_NB=$nb timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/sw.json 2>gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('NB=$nb', round(d['value'],1), {a:round(b,2) for a,b in k.items()})" || tail -5 gpurun_out/sw.err
done
