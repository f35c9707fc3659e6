mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -2 gpurun_out/t.log
timeout 400 python bench.py --cascade c6 --steps 3 --warmup 3 --no-cpu > gpurun_out/b_c6.json 2>gpurun_out/b_c6.err; tail -2 gpurun_out/b_c6.err
python -c "import json;d=json.load(open('gpurun_out/b_c6.json'));print('c6',round(d['value'],1),d['e2e']['value'],d['config']['workload'],{k:round(v,1) for k,v in d['kernel_ms_per_step'].items()})"
