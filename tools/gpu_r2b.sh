# f1 first light: quick parity, the full -m gpu suite, bench
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "depth_maps_bit_exact_small or worked_example or detections_identical" > gpurun_out/t_quick.log 2>&1; tail -15 gpurun_out/t_quick.log
timeout 2000 python -m pytest tests -m gpu -q > gpurun_out/t.log 2>&1; tail -25 gpurun_out/t.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/b.json 2>gpurun_out/b.err; tail -5 gpurun_out/b.err
cat gpurun_out/b.json
