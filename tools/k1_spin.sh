# K1 dataflow: __nanosleep back-off in the ready-byte polls (MP_K1_SPIN ns), twice each
# (experiment record: the code behind this knob was removed after the A/B measured it slower / neutral -- DESIGN "Experiments that did not pay")
set -u
for rep in 1 2; do for ns in 0 32 128 512; do
  MP_K1_SPIN=$ns timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/k1s_$ns.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/k1s_$ns.log').read().strip().splitlines()[-1]); k=d['roofline']['per_kernel_ms_per_step']; print('SPIN=$ns', round(d['ms_per_step'],3), k.get('k_rep2_bl<A>'))" || tail -3 gpurun_out/k1s_$ns.log
done; done
