#!/bin/bash
# Full measurement batch for one round (run under gpurun from the repo root).
# Writes everything under gpurun_out/meas/; tools/summarize.py copies it to profiles/<round>/.
set -u
O=gpurun_out/meas
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > $O/gpu.txt
timeout 900 python bench.py > $O/bench_c5.json 2> $O/bench_c5.err; echo "c5 rc=$?"
for R in 512 1024 2048; do
  timeout 300 python bench.py --replicas $R --no-cpu-baseline > $O/bench_c5_R$R.json 2> $O/bench_c5_R$R.err; echo "R$R rc=$?"
done
for c in c1 c2 c3 c4 c4fmm lu64 hier c2n4 c2push; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --cpu-budget-s 8 > $O/bench_$c.json 2> $O/bench_$c.err; echo "$c rc=$?"
done
for c in c5sim c5loc; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --cpu-budget-s 8 > $O/bench_$c.json 2> $O/bench_$c.err; echo "$c rc=$?"
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref_c5.json 2> $O/bench_ref.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c5.csv \
   python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-tlevel > $O/launches_c5.log 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rep2 -c 3 -o $O/full_c5 \
   python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-tlevel > $O/full_c5.log 2>&1; echo "full c5 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bl_small|k_sort_pass|k_kahn" -c 3 -o $O/full_c2 \
   python bench.py --config c2 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-probe --no-tlevel > $O/full_c2.log 2>&1; echo "full c2 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bl_flow|k_kahn|k_sort_pass" -c 4 -o $O/full_c4 \
   python bench.py --config c4 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-probe --no-tlevel > $O/full_c4.log 2>&1; echo "full c4 rc=$?"
