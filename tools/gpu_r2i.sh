mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/t.log 2>&1; tail -4 gpurun_out/t.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/b.json 2>gpurun_out/b.err; tail -3 gpurun_out/b.err
python -c "import json;d=json.load(open('gpurun_out/b.json'));print(d['value'],d['e2e']['value'],d['roofline']['kernel'],d['roofline']['frac'],d['kernel_ms_per_step_one_slot'])"
bash tools/gpu_sweep.sh "FD_F1=1" "FD_DEEP_SPLIT=0" 2>&1
