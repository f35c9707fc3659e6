# usage: TEST_ENV="..." CFGS='"A=1 B=2" "A=3"' bash tools/gpu_sweep2.sh -- parity tests under TEST_ENV, then bench per config
mkdir -p gpurun_out
if [ -n "$TEST_ENV" ]; then env $TEST_ENV timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log; fi
eval set -- $CFGS
for cfg in "$@"; do
  env $cfg timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/sw.json 2>gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$cfg', round(d['value'],1), {a:round(b,2) for a,b in k.items()})" || tail -3 gpurun_out/sw.err
done
