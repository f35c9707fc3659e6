mkdir -p gpurun_out
run() { # tag env... (extra bench args in BARGS)
  tag=$1; shift
  env "$@" timeout 400 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e $BARGS > gpurun_out/b_$tag.json 2>gpurun_out/b_$tag.err; tail -2 gpurun_out/b_$tag.err
  python -c "import json;d=json.load(open('gpurun_out/b_$tag.json'));k=d.get('kernel_ms_per_step_one_slot');print('$tag',round(d['value'],1),round(k['deep'],1),round(k.get('tail',0),1))"
}
run base
run t9 FD_DQ_TAIL=9
run t12 FD_DQ_TAIL=12
BARGS="--cascade c6" run c6
BARGS="--cascade c6" run c6t9 FD_DQ_TAIL=9
BARGS="--cascade c6" run c6d1 FD_DEEPQ=0
