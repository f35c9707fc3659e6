mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
run() { env FD_PIPE=0 "$@" timeout 300 python bench.py --frames 128 --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/sw.json 2>gpurun_out/sw.err || tail -3 gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$*',round(d['value'],1),{a:round(b,2) for a,b in k.items()})"; }
for S in 2 3 4 5 6 8; do run FD_S0=$S; done
run FD_S0=3 FD_S1_TAIL=0
run FD_S0=5 FD_S1_TAIL=0
