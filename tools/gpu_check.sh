# HEAD check on one B200: gpu tests, smoke, bench
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/t.log 2>&1; tail -4 gpurun_out/t.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/b.json 2>gpurun_out/b.err; tail -3 gpurun_out/b.err
python -c "import json;d=json.load(open('gpurun_out/b.json'));print(d['value'],d['e2e']['value'],d['roofline']['kernel'],d['roofline']['frac'],d['roofline_k2_other']['frac'],d.get('kernel_ms_per_step_one_slot'))"
for c in c6 c3s; do timeout 600 python bench.py --cascade $c --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/b_$c.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/b_$c.json'));print('$c',round(d['value'],1))"; done
