set -u
mkdir -p gpurun_out/p
for c in c2 c3 c4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/p/bench_$c.json 2> gpurun_out/p/bench_$c.err; echo "$c rc=$?"
done
timeout 600 python bench.py --steps 10 --warmup 3 --cpu-budget-s 8 > gpurun_out/p/bench_c5.json 2> gpurun_out/p/bench_c5.err; echo "c5 rc=$?"
nproc
