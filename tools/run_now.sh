mkdir -p gpurun_out/s36
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "replica or c5" > gpurun_out/s36/rep_tests.log 2>&1; rc=$?; echo tests=$rc; tail -2 gpurun_out/s36/rep_tests.log
if [ $rc -ne 0 ]; then exit 0; fi
VARS="head prio" RS="4096 2048 1024 512" bash tools/ab.sh
