# k_deepq bring-up: targeted parity, then bench (default and FD_DEEPQ=0)
mkdir -p gpurun_out
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/b_dq.json 2>gpurun_out/b_dq.err; tail -3 gpurun_out/b_dq.err
python -c "import json;d=json.load(open('gpurun_out/b_dq.json'));print('b_dq',round(d['value'],1),d.get('kernel_ms_per_step_one_slot'))"
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "k2_schedules or all_pass or bench_shape or small_groups or detections_identical or c6 or packed16 or soft_bench or step or ragged or min_size or many_levels" > gpurun_out/t_dq.log 2>&1; tail -15 gpurun_out/t_dq.log
