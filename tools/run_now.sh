mkdir -p gpurun_out/meas
for c in lu64 hier; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --cpu-budget-s 8 > gpurun_out/meas/bench_$c.json 2> gpurun_out/meas/bench_$c.err; echo "$c rc=$?"
done
