mkdir -p gpurun_out
run() { # tag env... (extra bench args in BARGS)
  tag=$1; shift
  env "$@" timeout 400 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e $BARGS > gpurun_out/b_$tag.json 2>gpurun_out/b_$tag.err; tail -2 gpurun_out/b_$tag.err
  python -c "import json;d=json.load(open('gpurun_out/b_$tag.json'));k=d.get('kernel_ms_per_step_one_slot');print('$tag',round(d['value'],1),round(k['deep'],1),round(k.get('tail',0),1),round(k['cascade'],1))"
}
run base
run j60 FD_JIT_DEEPQ_STUMPS=60
run j100 FD_JIT_DEEPQ_STUMPS=100
run j150 FD_JIT_DEEPQ_STUMPS=150
run g8 FD_DQ_GROUP=8
run g4 FD_DQ_GROUP=4
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_deepq" -c 1 -o gpurun_out/dq_def -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_dq.log 2>&1; tail -1 gpurun_out/ncu_dq.log
