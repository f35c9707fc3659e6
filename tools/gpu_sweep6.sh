mkdir -p gpurun_out
run() { env FD_PIPE=0 "$@" timeout 300 python bench.py --frames 128 --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/sw.json 2>gpurun_out/sw.err || tail -3 gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$*',round(d['value'],1),{a:round(b,2) for a,b in k.items()})"; }
run FD_JIT_DEEP_STUMPS=90
run FD_JIT_DEEP_STUMPS=60
run FD_JIT_DEEP_STUMPS=30
run FD_JIT_DEEP_STUMPS=14
run FD_JIT_DEEP_STUMPS=60 FD_TAIL_N=16
