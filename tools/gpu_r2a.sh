# round-2 baseline: gpu tests (incl. the bench-shape parity tests), smoke, bench
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
nproc > gpurun_out/nproc.txt; lscpu > gpurun_out/lscpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -rs -s -k "bench_shape or small_groups or 4k" > gpurun_out/t_new.log 2>&1; tail -5 gpurun_out/t_new.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
timeout 400 python bench.py --steps 5 --warmup 3 > gpurun_out/b.json 2>gpurun_out/b.err; tail -3 gpurun_out/b.err
head -c 600 gpurun_out/b.json
