mkdir -p gpurun_out/s28
cp ab/libmp_p640b8.so paper_conf_ipps_tayebbfg24_b200/libmp.so
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "configs_bit_exact or c4_bit or id_order" > gpurun_out/s28/quick.log 2>&1; rc=$?; echo quick=$rc; tail -2 gpurun_out/s28/quick.log
if [ $rc -ne 0 ]; then exit 0; fi
for rep in 1 2; do for v in p1024b4 p1024b5 p768b6 p640b8; do
  cp ab/libmp_$v.so paper_conf_ipps_tayebbfg24_b200/libmp.so
  for c in c3 c4 c4fmm; do echo "== $v $(timeout 120 python tools/ingest_breakdown.py $c 10 2>&1 | head -1 | cut -c1-60)"; done
done; done
cp ab/libmp_p1024b4.so paper_conf_ipps_tayebbfg24_b200/libmp.so
