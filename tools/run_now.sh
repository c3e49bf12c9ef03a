mkdir -p gpurun_out/s27
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "configs_bit_exact or c4_bit or id_order or deep_chain" > gpurun_out/s27/quick.log 2>&1; rc=$?; echo quick=$rc; tail -2 gpurun_out/s27/quick.log
if [ $rc -ne 0 ]; then exit 0; fi
for rep in 1 2; do for v in head rf2; do
  cp ab/libmp_$v.so paper_conf_ipps_tayebbfg24_b200/libmp.so
  for c in c2 c3 c4 c4fmm; do echo "== $v $(timeout 120 python tools/ingest_breakdown.py $c 10 2>&1 | head -1 | cut -c1-50) $(timeout 120 python tools/ingest_breakdown.py $c 10 2>&1 | head -1 | grep -o "'k_rcsr_fill': [0-9.]*")"; done
done; done
cp ab/libmp_rf2.so paper_conf_ipps_tayebbfg24_b200/libmp.so
