mkdir -p gpurun_out/s16
cp ab/libmp_kid0.so paper_conf_ipps_tayebbfg24_b200/libmp.so
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/s16/gpu_tests_kid0.log 2>&1; echo tests_kid0=$?; tail -2 gpurun_out/s16/gpu_tests_kid0.log
cp ab/libmp_kid.so paper_conf_ipps_tayebbfg24_b200/libmp.so
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/s16/gpu_tests_kid.log 2>&1; echo tests_kid=$?; tail -2 gpurun_out/s16/gpu_tests_kid.log
for v in flow2 kid kid0 kidb8; do
  cp ab/libmp_$v.so paper_conf_ipps_tayebbfg24_b200/libmp.so
  for c in c2 lu64 c3 c4; do echo "== $v"; timeout 300 python tools/ingest_breakdown.py $c 5 2>&1 | head -1 | cut -c1-200; done
done
cp ab/libmp_kid.so paper_conf_ipps_tayebbfg24_b200/libmp.so
