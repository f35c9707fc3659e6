mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
timeout 300 python tools/k2_timing.py > gpurun_out/k2t.txt 2>&1; head -4 gpurun_out/k2t.txt
timeout 300 python bench.py --steps 5 --warmup 3 > gpurun_out/b.json 2>gpurun_out/b.err
python -c "import json;d=json.load(open('gpurun_out/b.json'));print(d['value'],d['e2e']['value'],d['kernel_ms_per_step'])"
