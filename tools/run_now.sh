mkdir -p gpurun_out/s31
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/s31/gpu_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/s31/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()"; echo smoke=$?
