mkdir -p gpurun_out
( for cfg in "X=1" "X=2" "X=3" "X=4" "X=5" "X=6"; do
  echo "== $cfg"; env $cfg timeout 120 python tools/repro_c6q.py 32 > gpurun_out/r.txt 2>&1; echo "rc=$?"; tail -n 1 gpurun_out/r.txt
done ) > gpurun_out/dbg.txt 2>&1
cat gpurun_out/dbg.txt
