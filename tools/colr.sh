# one-block Kahn with per-edge target ranges (MP_KAHN_COLR) + k_bl_small L2 prefetch: parity, A/B, c2/c5 lines
set -u
mkdir -p gpurun_out/cr
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/cr/gpu_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/cr/gpu_tests.log
for cr in 0 1; do echo "== COLR=$cr c2"; MP_KAHN_COLR=$cr timeout 300 python tools/ingest_breakdown.py c2 5 2>&1 | tail -2 | cut -c1-200; done
for c in c2; do
timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/cr/bench_$c.json 2> gpurun_out/cr/bench_$c.err; echo $c=$?
python -c "import json;d=json.loads(open('gpurun_out/cr/bench_$c.json').read().strip().splitlines()[-1]);print(d['ms_per_step'], d['score_only']['ms_per_dag'], d['roofline']['per_kernel_ms_per_step'])" | cut -c1-400
done
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/cr/bench_c5.json 2> gpurun_out/cr/bench_c5.err; echo c5=$?
python -c "import json;d=json.loads(open('gpurun_out/cr/bench_c5.json').read().strip().splitlines()[-1]);print(d['ms_per_step'], d['roofline']['per_kernel_ms_per_step'])" | cut -c1-300
