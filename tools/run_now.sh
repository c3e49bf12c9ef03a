mkdir -p gpurun_out/s21
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/s21/gpu_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/s21/gpu_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/s21/bench_c5.json 2>gpurun_out/s21/bench_c5.err; python -c "
import json; d=json.loads(open('gpurun_out/s21/bench_c5.json').read().strip().splitlines()[-1]); print('c5', round(d['ms_per_step'],3), d.get('build_ms'), d['e2e']['value'])"
for c in c2 c3 c4; do timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/s21/bench_$c.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/s21/bench_$c.json').read().strip().splitlines()[-1]); print('$c', round(d['ms_per_step'],3), 'build', round(d['build_ms'],3))"; done
