# k_kahn<SF> templated, late range loads by default: parity + single-DAG bench lines + c5
set -u
mkdir -p gpurun_out/kf
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/kf/parity.log 2>&1; echo parity=$?; tail -1 gpurun_out/kf/parity.log
for c in c2 c3 c4 lu64; do
timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-probe > gpurun_out/kf/bench_$c.json 2> gpurun_out/kf/bench_$c.err
python -c "import json;d=json.loads(open('gpurun_out/kf/bench_$c.json').read().strip().splitlines()[-1]);k=d['roofline']['per_kernel_ms_per_step'];print('$c', round(d['ms_per_step'],3), {x:k[x] for x in k if 'kahn' in x})"
done
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/kf/bench_c5.json 2> gpurun_out/kf/bench_c5.err
python -c "import json;d=json.loads(open('gpurun_out/kf/bench_c5.json').read().strip().splitlines()[-1]);k=d['roofline']['per_kernel_ms_per_step'];print('c5', round(d['ms_per_step'],3), {x:k[x] for x in k if 'kahn' in x})"
