#!/bin/bash
# session start check (run under gpurun): GPU tests at HEAD, c5 bench, source-level ncu of K1/K2
set -u
O=gpurun_out/s3
mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q -x > $O/gpu_tests.log 2>&1; echo tests=$?; tail -3 $O/gpu_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_c5.json 2> $O/bench_c5.err; echo bench=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rep2 -c 2 -o $O/full_c5 -f \
   python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-tlevel > $O/full_c5.log 2>&1; echo "full c5 rc=$?"
