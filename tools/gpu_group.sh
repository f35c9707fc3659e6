mkdir -p gpurun_out
timeout 300 python tools/group_probe.py
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_group|k_seg" --csv --log-file gpurun_out/glaunch.csv python tools/group_probe.py > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/glaunch.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
for r in rows[-7:]: print(r[ki][:40], r[vi])
PY
