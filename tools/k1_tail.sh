# K1 flow mode: tail successors 4 at a time (MP_K1_FLOW=2) vs one at a time (1), twice each; parity under 2
# (experiment record: the code behind this knob was removed after the A/B measured it slower / neutral -- DESIGN "Experiments that did not pay")
set -u
for rep in 1 2; do for f in 1 2; do
  MP_K1_FLOW=$f timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/k1t_$f.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/k1t_$f.log').read().strip().splitlines()[-1]); k=d['roofline']['per_kernel_ms_per_step']; print('FLOW=$f', round(d['ms_per_step'],3), k.get('k_rep2_bl<A>'))" || tail -3 gpurun_out/k1t_$f.log
done; done
MP_K1_FLOW=2 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k replicas 2>&1 | tail -1
