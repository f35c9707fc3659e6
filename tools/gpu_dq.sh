mkdir -p gpurun_out
run() { # tag env... (extra bench args in BARGS)
  tag=$1; shift
  env "$@" timeout 400 python bench.py --steps 15 --warmup 3 --no-cpu --no-e2e $BARGS > gpurun_out/b_$tag.json 2>gpurun_out/b_$tag.err; tail -2 gpurun_out/b_$tag.err
  python -c "import json;d=json.load(open('gpurun_out/b_$tag.json'));k=d.get('kernel_ms_per_step_one_slot');print('$tag',round(d['value'],1),round(k['deep'],1),round(k.get('tail',0),1),round(k['cascade'],1))"
}
run d1 FD_DEEPQ=0
run q255 FD_DEEPQ=1 FD_DQ_TAIL=255
run q9 FD_DEEPQ=1 FD_DQ_TAIL=9
run d1b FD_DEEPQ=0
run q255b FD_DEEPQ=1 FD_DQ_TAIL=255
BARGS="--cascade c6" run c6d1 FD_DEEPQ=0
BARGS="--cascade c6" run c6q255 FD_DEEPQ=1 FD_DQ_TAIL=255
BARGS="--cascade c6" run c6q9 FD_DEEPQ=1 FD_DQ_TAIL=9
