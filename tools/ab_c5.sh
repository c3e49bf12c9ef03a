#!/bin/bash
# A/B of the c5 bench under an env toggle: tools/ab_c5.sh VAR  (runs VAR=0 then default)
for v in 0 1; do
  if [ $v = 0 ]; then export $1=0; else unset $1; fi
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab_$v.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/ab_$v.log').read().strip().splitlines()[-1]); k=d['roofline']['per_kernel_ms_per_step']; print('$1=$v', round(d['ms_per_step'],3), k.get('k_rep2_sort<A>'), k.get('k_rep2_bl<A>'))" || tail -3 gpurun_out/ab_$v.log
done
