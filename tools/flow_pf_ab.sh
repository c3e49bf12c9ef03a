#!/bin/bash
# k_bl_flow A/B over (edges per lane in flight, min blocks per SM): rebuilds libmp.so in the
# box's copy; prints the score-path time and k_bl_flow per config
set -u
O=gpurun_out/flowpf; mkdir -p $O
for v in "2 8" "4 4" "8 2" "8 4"; do
  set -- $v
  python -c "
import subprocess,sys; sys.path.insert(0,'paper_conf_ipps_tayebbfg24_b200'); import build as B
subprocess.check_call([B.NVCC,*B.FLAGS,'-DMP_FLOW_PF=$1','-DMP_FLOW_MINB=$2','-o',B.LIB,B.os.path.join(B.CSRC,'libmp.cu')])"
  for c in ${CFGS:-c4 c4fmm hier c3}; do
    timeout 300 python bench.py --config $c --steps 10 --no-cpu-baseline --no-e2e --no-probe > $O/pf$1_$2_$c.json 2>/dev/null
    python -c "
import json; d=json.loads(open('$O/pf$1_$2_$c.json').read().strip().splitlines()[-1]); k=d['roofline']['per_kernel_ms_per_step']
print('PF=$1 MINB=$2 $c', round(d['ms_per_step'],3), 'k_bl_flow', k.get('k_bl_flow'))"
  done
done
