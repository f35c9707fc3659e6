# ncu --set full of one k_deep launch (16 1080p frames), generic build (source-mapped)
mkdir -p gpurun_out
FD_JIT=0 timeout 300 python bench.py --frames 64 --steps 3 --warmup 1 --no-e2e --no-cpu > gpurun_out/gen.json 2>&1
python -c "import json;d=json.load(open('gpurun_out/gen.json'));print({a:round(b,2) for a,b in d['kernel_ms_per_step'].items()})"
FD_JIT=0 timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_deep -c 1 -o gpurun_out/deep_gen -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_deep.log 2>&1
tail -n 3 gpurun_out/ncu_deep.log
