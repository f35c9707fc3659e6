# Bench A/B sweep on one B200: each argument is a set of environment settings for one run, e.g.
#   bash tools/gpu_sweep.sh "FD_TAIL_N=8" "FD_TAIL_N=32" "FD_F1=0"
# FRAMES (default 512) frames per step, 3 timed steps, 2 warm-up; prints fps and the one-slot
# per-kernel ms of the untimed profiling pass.
mkdir -p gpurun_out
for cfg in "$@"; do
  env $cfg timeout 300 python bench.py --frames "${FRAMES:-512}" --steps 3 --warmup 2 --no-cpu --no-e2e \
    > gpurun_out/sw.json 2> gpurun_out/sw.err || tail -3 gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));k=d['kernel_ms_per_step_one_slot'];print('$cfg', round(d['value'],1), {a: round(b, 2) for a, b in k.items()})"
done
