# k_bl_small (weights prologue + next-level row prefetch): GPU tests, c2 and c5 bench lines
set -u
mkdir -p gpurun_out/bs
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/bs/gpu_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/bs/gpu_tests.log
for c in c2 lu64; do
timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bs/bench_$c.json 2> gpurun_out/bs/bench_$c.err; echo $c=$?
python -c "import json;d=json.loads(open('gpurun_out/bs/bench_$c.json').read().strip().splitlines()[-1]);print(d['ms_per_step'], d.get('score_only'), d['roofline']['per_kernel_ms_per_step'])" | cut -c1-600
done
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bs/bench_c5.json 2> gpurun_out/bs/bench_c5.err; echo c5=$?
python -c "import json;d=json.loads(open('gpurun_out/bs/bench_c5.json').read().strip().splitlines()[-1]);print(d['ms_per_step'], d['roofline']['per_kernel_ms_per_step'])"
