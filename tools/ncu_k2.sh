#!/bin/bash
# ncu --set full (with source) of one k_rep2_sort launch -> gpurun_out/full_k2.ncu-rep
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rep2_sort -c 1 -o gpurun_out/full_k2 -f \
   python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/full_k2.log 2>&1; echo "full k2 rc=$?"
