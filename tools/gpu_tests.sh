#!/bin/bash
# GPU test suite only (run under gpurun): gpurun_out/<tag>/gpu_tests.log
set -u
O=gpurun_out/${1:-t}
mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q ${2:-} > $O/gpu_tests.log 2>&1; echo tests=$?; tail -5 $O/gpu_tests.log
