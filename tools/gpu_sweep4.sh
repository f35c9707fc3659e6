mkdir -p gpurun_out
run() { env FD_PIPE=0 "$@" timeout 300 python bench.py --frames 128 --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/sw.json 2>gpurun_out/sw.err || tail -3 gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step'];print('$*',round(d['value'],1),round(k['cascade'],2),round(k['deep'],2),round(k['tail'],2))"; }
run FD_K2_DEEP1=1
for NB in 1 2 4 8; do run FD_K2_DEEP1=0 FD_K2B_NB=$NB; done
run FD_K2_DEEP1=0 FD_K2B_NB=4 FD_TAIL_N=32
run FD_S0=1
