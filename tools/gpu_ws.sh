mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -5 gpurun_out/t.log
run() { env FD_PIPE=0 "$@" timeout 300 python bench.py --frames 128 --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/sw.json 2>gpurun_out/sw.err || tail -3 gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$*',round(d['value'],1),{a:round(b,2) for a,b in k.items()})"; }
run FD_K2_WS=1
run FD_K2_WS=0
run FD_K2_WS=1 FD_WS_DEEP_WARPS=4
run FD_K2_WS=1 FD_WS_S0=1 FD_WS_DEEP_WARPS=4
run FD_K2_WS=1 FD_WS_DEEP_WARPS=6
