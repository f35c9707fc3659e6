mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "k2_schedules or depth_maps or detections or video" > gpurun_out/t.log 2>&1; tail -2 gpurun_out/t.log
run() { env "$@" timeout 300 python bench.py --frames 512 --steps 3 --warmup 2 --no-cpu --no-e2e > gpurun_out/sw.json 2>gpurun_out/sw.err || tail -3 gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$*',round(d['value'],1),{a:round(b,2) for a,b in k.items()})"; }
run FD_PIPE=0
run FD_PIPE=0 FD_K2D_CTAS=4
run FD_PIPE=1
