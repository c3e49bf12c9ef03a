#!/bin/bash
# compute-sanitizer: memcheck / racecheck / synccheck / initcheck on the small run and the
# large one (gpurun_out/san2/*.log); exit lines summarised
O=gpurun_out/san2; mkdir -p $O
for tool in memcheck racecheck synccheck initcheck; do
  for run in sanitize_run sanitize_large; do
    timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/$run.py > $O/${tool}_${run}.log 2>&1
    echo "$tool $run rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|run ok' $O/${tool}_${run}.log | tr '\n' ' ')"
  done
done
