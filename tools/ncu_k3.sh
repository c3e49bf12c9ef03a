#!/bin/bash
# ncu --set full (with source) of one k_rep3_sort launch -> gpurun_out/<tag>/full_k3.ncu-rep
O=gpurun_out/${1:-k3}
mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rep3_sort -c 1 -o $O/full_k3 -f \
   python bench.py --steps 1 --warmup 0 --replicas ${2:-592} --no-cpu-baseline --no-e2e > $O/full_k3.log 2>&1; echo "full k3 rc=$?"
