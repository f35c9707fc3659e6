# usage: bash tools/gpu_sweep.sh VAR v1 v2 ... -- bench K2 ms per setting of an env variable
var=$1; shift
mkdir -p gpurun_out
for v in "$@"; do
  env $var=$v timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/sw.json 2>gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$var=$v', round(d['value'],1), {a:round(b,2) for a,b in k.items()})" || tail -5 gpurun_out/sw.err
done
