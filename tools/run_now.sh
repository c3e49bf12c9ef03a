mkdir -p gpurun_out/s33
cp ab/libmp_lpt.so paper_conf_ipps_tayebbfg24_b200/libmp.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "replica or c5" > gpurun_out/s33/rep_tests.log 2>&1; rc=$?; echo tests=$rc; tail -2 gpurun_out/s33/rep_tests.log
if [ $rc -ne 0 ]; then exit 0; fi
VARS="head lpt" RS="4096 2048 1024 512" bash tools/ab.sh
