#!/bin/bash
# Same-box A/B of prebuilt libmp variants (run under gpurun): ab/libmp_<v>.so for v in $VARS,
# each copied over the in-tree libmp.so, c5 bench at R = 4096 (and $RS), twice, interleaved.
set -u
O=gpurun_out/ab; mkdir -p $O
cp paper_conf_ipps_tayebbfg24_b200/libmp.so ab/libmp_orig.so
for rep in 1 2; do
  for v in ${VARS:-base new}; do
    cp ab/libmp_$v.so paper_conf_ipps_tayebbfg24_b200/libmp.so
    for R in ${RS:-4096}; do
      timeout 300 python bench.py --replicas $R --steps 10 --no-cpu-baseline --no-e2e --no-tlevel ${BENCH_ARGS:-} > $O/${v}_R${R}_$rep.json 2>$O/${v}_R${R}_$rep.err
      python -c "
import json; d=json.loads(open('$O/${v}_R${R}_$rep.json').read().strip().splitlines()[-1]); k=d['roofline']['per_kernel_ms_per_step']
print('$v R=$R rep=$rep', round(d['ms_per_step'],3), {a: round(b,3) for a,b in k.items()})" || tail -3 $O/${v}_R${R}_$rep.err
    done
  done
done
cp ab/libmp_orig.so paper_conf_ipps_tayebbfg24_b200/libmp.so
