mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_dist.py -m gpu -q -k "host or group or smoke or dist or rank or bench_shape" > gpurun_out/t_h2d.log 2>&1; tail -2 gpurun_out/t_h2d.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu > gpurun_out/b_h2d.json 2>gpurun_out/b_h2d.err; tail -2 gpurun_out/b_h2d.err
python -c "import json;d=json.load(open('gpurun_out/b_h2d.json'));print('h2d',round(d['value'],1),d['e2e'])"
