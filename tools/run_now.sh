mkdir -p gpurun_out/s35
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/s35/gpu_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/s35/gpu_tests.log
echo "== $(timeout 300 python tools/bl_time.py c2 lu64 hier 2>&1 | tail -3 | tr '\n' ' ' | cut -c1-250)"
