# HEAD check on one B200: gpu tests, smoke, bench
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/t_head.log 2>&1; tail -3 gpurun_out/t_head.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/b_head.json 2>gpurun_out/b_head.err; tail -2 gpurun_out/b_head.err
python -c "import json;d=json.load(open('gpurun_out/b_head.json'));print(d['value'],d['e2e']['value'],d['roofline']['frac'],d['roofline_k2_other']['frac'],d['roofline_k2_other']['traffic'],d.get('kernel_ms_per_step_one_slot'))"
