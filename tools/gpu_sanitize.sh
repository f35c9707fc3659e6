# compute-sanitizer (memcheck, racecheck, synccheck) on the small all-kernel workload; summaries to gpurun_out/
mkdir -p gpurun_out
for mode in default f1; do
  if [ $mode = f1 ]; then export FD_F1=1; else unset FD_F1; fi
  for tool in memcheck racecheck synccheck; do
    timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_case.py > gpurun_out/san_${mode}_${tool}.txt 2>&1
    echo "$mode $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' gpurun_out/san_${mode}_${tool}.txt | tail -n 2 | tr '\n' ' ')"
  done
done
