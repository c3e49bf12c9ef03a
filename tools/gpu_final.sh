#!/bin/bash
# round-end batch: GPU tests, smoke, the measurement batch (tools/measure.sh)
set -u
mkdir -p gpurun_out/meas
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/meas/gpu_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/meas/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/meas/smoke.log 2>&1; echo "smoke rc=$?"
bash tools/measure.sh
