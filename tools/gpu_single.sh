#!/bin/bash
# single-DAG parity tests + score-only times of c3 / c4 / lu64 (run under gpurun)
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_n4.py -x -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo tests=$?; tail -1 gpurun_out/gpu_tests.log
for c in ${@:-c3 c4 lu64}; do
  timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/so_$c.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/so_$c.log').read().strip().splitlines()[-1]); s=d['score_only']; k=d['roofline']['per_kernel_ms_per_step']
print('$c', 'step', round(d['ms_per_step'],3), 'score', round(s['ms_per_dag'],3), 'bl_flow', k.get('k_bl_flow'), 'kahn', k.get('k_kahn'))" || tail -3 gpurun_out/so_$c.log
done
