# final round-2 measurements on one B200: every GPU test, smoke, the bench (+ variants and the
# reference arm), ncu launch list, ncu --set full of the path's kernels, L2 bytes; all in gpurun_out/
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/t_final.log 2>&1; tail -3 gpurun_out/t_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/b_final.json 2>gpurun_out/b_final.err; tail -n 2 gpurun_out/b_final.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/b_ref.json 2>gpurun_out/b_ref.err
for c in c3s c6 c6q; do timeout 600 python bench.py --cascade $c --steps 5 --warmup 3 --no-cpu > gpurun_out/b_$c.json 2>gpurun_out/b_$c.err; done
FD_DEEPQ=0 timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/b_deep1.json 2>gpurun_out/b_deep1.err
FD_F1=1 timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/b_f1.json 2>gpurun_out/b_f1.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_r2c.csv \
  python bench.py --frames 256 --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/ncu_l.log 2>&1; tail -1 gpurun_out/ncu_l.log
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_stage1|k_deepq|k_marg|k_carry|k_corner|k_tile|k_group" -c 9 -o gpurun_out/full_r2c -f \
  python bench.py --frames 128 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1; tail -1 gpurun_out/ncu_full.log
timeout 900 ncu --metrics lts__t_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"k_stage1|k_deepq|k_marg|k_tile" -c 8 --csv --log-file gpurun_out/l2_r2c.csv \
  python bench.py --frames 128 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_l2.log 2>&1
for f in b_final b_ref b_c3s b_c6 b_c6q b_deep1 b_f1; do python -c "import json;d=json.load(open('gpurun_out/$f.json'));print('$f', round(d['value'],1), d.get('e2e',{}).get('value'), d.get('c3_single_frame',{}).get('frames_per_s'))"; done
