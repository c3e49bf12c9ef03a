#!/bin/bash
# one ncu --set full capture (with source) of the two c5 replica kernels -> gpurun_out/full_c5.ncu-rep
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rep2 -c 2 -o gpurun_out/full_c5 -f \
   python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/full_c5.log 2>&1; echo "full c5 rc=$?"
ls -la gpurun_out/
