# split-K2 check: GPU parity, then bench per configuration (CFGS env overrides the list)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
for cfg in ${CFGS:-"FD_K2_SPLIT=0" "FD_K2B_NB=2" "FD_K2B_NB=4" "FD_K2B_NB=6" "FD_K2B_NB=8" "FD_K2B_NB=4 FD_TAIL_N=16" "FD_K2B_NB=8 FD_TAIL_N=32"}; do
  env $cfg timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/sw.json 2>gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$cfg', round(d['value'],1), {a:round(b,2) for a,b in k.items()})" || tail -5 gpurun_out/sw.err
done
