mkdir -p gpurun_out/s17
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "replica or c5" > gpurun_out/s17/rep_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/s17/rep_tests.log
VARS="eq2 k2fast" RS="4096 512" bash tools/ab.sh
