mkdir -p gpurun_out/meas
timeout 900 python bench.py > gpurun_out/meas/bench_c5.json 2> gpurun_out/meas/bench_c5.err; echo "c5 rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/meas/bench_c5.json').read().strip().splitlines()[-1]); r=d['roofline']; print(d['ms_per_step'], d['value'], r['frac'], r['per_kernel_ms_per_step'])"
