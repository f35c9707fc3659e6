mkdir -p gpurun_out
run() { # tag env... (extra bench args in BARGS)
  tag=$1; shift
  env "$@" timeout 400 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e $BARGS > gpurun_out/b_$tag.json 2>gpurun_out/b_$tag.err; tail -2 gpurun_out/b_$tag.err
  python -c "import json;d=json.load(open('gpurun_out/b_$tag.json'));k=d.get('kernel_ms_per_step_one_slot');print('$tag',round(d['value'],1),round(k['deep'],1),round(k.get('tail',0),1),round(k['cascade'],1))"
}
run q255w32 FD_DEEPQ=1 FD_DQ_TAIL=255 FD_DQ_WARPS=32
run q255w24 FD_DEEPQ=1 FD_DQ_TAIL=255 FD_DQ_WARPS=24
run q9w32 FD_DEEPQ=1 FD_DQ_TAIL=9 FD_DQ_WARPS=32
run q255w32s12 FD_DEEPQ=1 FD_DQ_TAIL=255 FD_DQ_WARPS=32 FD_DQ_SLOTS=12
run b7w32 FD_DEEPQ=2 FD_DQ_TAIL=9 FD_DB_WARPS=32
