# K2 marginal cost per stage: c3 truncated to its first k stages (depth mode), per tiles-per-batch setting
mkdir -p gpurun_out
for nb in ${NBS:-1 3}; do
  echo "NB=$nb"; FD_K2_NB=$nb timeout 300 python tools/k2_truncate.py r1:10 1 2 3 4 5 6 8 10 15 25
done
