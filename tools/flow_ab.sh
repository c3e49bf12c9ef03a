#!/bin/bash
# k_bl_flow variants: prefetch depth x min blocks per SM (rebuilds libmp.so in place on the box), 3 runs each
for v in ${FLOW_VARIANTS:-"2 8" "4 8" "8 1"}; do
  set -- $v
  python -c "
from paper_conf_ipps_tayebbfg24_b200 import build as B; import subprocess,os
subprocess.check_call([B.NVCC,*B.FLAGS,'-DMP_FLOW_PF=$1','-DMP_FLOW_MINB=$2','-o',B.LIB,os.path.join(B.CSRC,'libmp.cu')])"
  for c in c3 c4 lu64; do
    for rep in 1 2 3; do
    timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/fa_$c.log 2>&1
    python -c "
import json; d=json.loads(open('gpurun_out/fa_$c.log').read().strip().splitlines()[-1]); k=d['roofline']['per_kernel_ms_per_step']
print('pf=$1 minb=$2 $c', 'score', round(d['score_only']['ms_per_dag'],3), 'bl_flow', k.get('k_bl_flow'))"
    done
  done
done
