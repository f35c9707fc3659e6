mkdir -p gpurun_out
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e > gpurun_out/b_gp.json 2>gpurun_out/b_gp.err; tail -2 gpurun_out/b_gp.err
python -c "import json;d=json.load(open('gpurun_out/b_gp.json'));k=d.get('kernel_ms_per_step_one_slot');print('gp',round(d['value'],1),{a:round(b,1) for a,b in k.items()})"
timeout 300 python bench.py --cascade c6 --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/b_gp_c6.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/b_gp_c6.json'));k=d.get('kernel_ms_per_step_one_slot');print('gp c6',round(d['value'],1),round(k['deep'],1))"
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "k2_schedules or all_pass or bench_shape or default_groups or c6_workload" > gpurun_out/t_gp.log 2>&1; tail -2 gpurun_out/t_gp.log
