#!/bin/bash
# round-2 batch: GPU tests, smoke, c5 headline + 1-GPU strong-scaling proxies, single-DAG lines
set -u
O=gpurun_out/${1:-r2a}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt
timeout 1800 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; echo tests=$?; tail -3 $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 600 python bench.py > $O/bench_c5.json 2> $O/bench_c5.err; echo c5=$?
for R in 512 1024 2048; do
  timeout 300 python bench.py --replicas $R --no-cpu-baseline --no-e2e > $O/bench_c5_R$R.json 2> $O/bench_c5_R$R.err; echo R$R=$?
done
for c in c2 c4fmm c4; do
  timeout 600 python bench.py --config $c --steps 10 --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?
done
