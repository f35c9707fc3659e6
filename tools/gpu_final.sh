# final measurements: bench (default + variants), ncu launch list and full capture, summaries in gpurun_out/
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/b_final.json 2>gpurun_out/b_final.err; tail -n 2 gpurun_out/b_final.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/b_ref.json 2>gpurun_out/b_ref.err
for c in c3s c6 c6q; do timeout 600 python bench.py --cascade $c --steps 5 --warmup 3 --no-cpu > gpurun_out/b_$c.json 2>gpurun_out/b_$c.err; done
FD_F1=1 timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/b_f1.json 2>gpurun_out/b_f1.err
TAG=r2 KRE="k_stage1|k_deep1|k_tail|k_marg|k_carry|k_corner|k_tile|k_group|k_keys" NK=14 bash tools/gpu_ncu_r2.sh
timeout 900 ncu --metrics lts__t_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"k_stage1|k_deep1|k_tail|k_marg|k_tile|k_f1|k_level" -c 12 --csv --log-file gpurun_out/l2_r2.csv \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_l2.log 2>&1
FD_F1=1 timeout 900 ncu --set full --clock-control none -k regex:"k_f1|k_level|k_deep1|k_tail" -c 4 -o gpurun_out/full_f1_r2 -f \
  python bench.py --frames 16 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_f1.log 2>&1
for f in b_final b_ref b_c3s b_c6 b_c6q b_f1; do python -c "import json;d=json.load(open('gpurun_out/$f.json'));print('$f', round(d['value'],1), d.get('e2e',{}).get('value'))"; done
