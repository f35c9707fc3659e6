mkdir -p gpurun_out
for TN in 8 16 32 64 128 256; do
  FD_PIPE=0 FD_TAIL_N=$TN timeout 300 python bench.py --frames 128 --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/sw.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('tail_n $TN',round(d['value'],1),round(k['cascade'],2),round(k['deep'],2),round(k['tail'],2))"
done
for C in 4 8; do
  FD_PIPE=0 FD_K2D_CTAS=$C timeout 300 python bench.py --frames 128 --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/sw.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('ctas $C',round(d['value'],1),round(k['cascade'],2),round(k['deep'],2),round(k['tail'],2))"
done
FD_PIPE=0 MODE=detect timeout 300 python tools/k2_truncate.py 1 2 3 4 5 6 8 12 25 > gpurun_out/trunc.txt 2>&1; cat gpurun_out/trunc.txt
