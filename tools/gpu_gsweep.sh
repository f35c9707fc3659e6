mkdir -p gpurun_out
run() { env "$@" timeout 300 python bench.py --frames 512 --steps 3 --warmup 2 --no-cpu --no-e2e > gpurun_out/sw.json 2>gpurun_out/sw.err || tail -3 gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$*',round(d['value'],1),{a:round(b,2) for a,b in k.items()})"; }
for G in 16 32 64 128; do run FD_GROUP_FRAMES=$G; done
run FD_GROUP_FRAMES=64 FD_PIPE=0
