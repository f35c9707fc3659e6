mkdir -p gpurun_out
run() { # tag env...
  tag=$1; shift
  env "$@" timeout 400 python bench.py --steps 8 --warmup 3 --no-cpu --no-e2e > gpurun_out/b_$tag.json 2>gpurun_out/b_$tag.err; tail -2 gpurun_out/b_$tag.err
  python -c "import json;d=json.load(open('gpurun_out/b_$tag.json'));k=d.get('kernel_ms_per_step_one_slot');print('$tag',round(d['value'],1),{a:round(b,1) for a,b in k.items()})"
}
run g16 FD_GROUP_FRAMES=16
run g32 FD_GROUP_FRAMES=32
run g64 FD_GROUP_FRAMES=64
run g128 FD_GROUP_FRAMES=128
run g256 FD_GROUP_FRAMES=256
run g16b FD_GROUP_FRAMES=16
timeout 600 python bench.py --cascade c6q --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/b_c6q2.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/b_c6q2.json'));print('c6q',round(d['value'],1))"
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "c6q or packed16" > gpurun_out/t_c6q.log 2>&1; tail -1 gpurun_out/t_c6q.log
