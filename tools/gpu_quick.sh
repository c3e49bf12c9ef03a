#!/bin/bash
# quick GPU check: replica parity tests + c5 bench summary (run under gpurun)
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "${1:-replica}" > gpurun_out/gpu_tests.log 2>&1; echo tests=$?; tail -3 gpurun_out/gpu_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline ${2} > gpurun_out/bench_q.log 2>&1; echo bench=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench_q.log').read().strip().splitlines()[-1]); print(round(d['ms_per_step'],3), d['roofline']['per_kernel_ms_per_step'])" || tail -5 gpurun_out/bench_q.log
