mkdir -p gpurun_out
FD_DQ_SLOTS=2 FD_DQ_WARPS=4 timeout 120 python tools/dq_debug.py > gpurun_out/dbg_2s.log 2>&1; tail -3 gpurun_out/dbg_2s.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/b_dq.json 2>gpurun_out/b_dq.err; tail -3 gpurun_out/b_dq.err
python -c "import json;d=json.load(open('gpurun_out/b_dq.json'));print('b_dq',round(d['value'],1),d.get('kernel_ms_per_step_one_slot'))"
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "k2_schedules or all_pass or bench_shape" > gpurun_out/t_dq.log 2>&1; tail -5 gpurun_out/t_dq.log
