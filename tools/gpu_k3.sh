#!/bin/bash
# K3 bring-up: replica parity tests (first failure stops), then a short c5 bench
set -u
O=gpurun_out/${1:-k3}
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "replica" > $O/tests.log 2>&1; echo tests=$?; tail -15 $O/tests.log
timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e > $O/bench_c5.json 2> $O/bench_c5.err; echo c5=$?; tail -3 $O/bench_c5.err
python -c "
import json; d=json.loads(open('$O/bench_c5.json').read().strip().splitlines()[-1]); r=d['roofline']
print('ms/step', d['ms_per_step'], r['per_kernel_ms_per_step'])"
