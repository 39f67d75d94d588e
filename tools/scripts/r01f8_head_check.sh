# HEAD of the round: GPU suite + smoke
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01f8_gpu_tests.log 2>&1; echo tests=$?
tail -2 gpurun_out/r01f8_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01f8_smoke.log 2>&1; echo smoke=$?
tail -1 gpurun_out/r01f8_smoke.log
