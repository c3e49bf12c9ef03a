#!/bin/bash
# K1 successor gathers in flight per lane (MP_K1_PF): c5 at R = 512 (strong-scaling proxy)
# and R = 4096 per variant; rebuilds libmp.so in the box's copy
set -u
O=gpurun_out/k1ab; mkdir -p $O
for pf in ${PFS:-8 16 32}; do
  python -c "
import subprocess,sys; sys.path.insert(0,'paper_conf_ipps_tayebbfg24_b200'); import build as B
subprocess.check_call([B.NVCC,*B.FLAGS,'-DMP_K1_PF=$pf','-o',B.LIB,B.os.path.join(B.CSRC,'libmp.cu')])"
  for R in 512 4096; do
    timeout 300 python bench.py --replicas $R --steps 10 --no-cpu-baseline --no-e2e --no-tlevel > $O/pf${pf}_R$R.json 2>/dev/null
    python -c "
import json; d=json.loads(open('$O/pf${pf}_R$R.json').read().strip().splitlines()[-1]); k=d['roofline']['per_kernel_ms_per_step']
print('PF=$pf R=$R', round(d['ms_per_step'],3), k)"
  done
done
