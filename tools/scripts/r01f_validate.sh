# re-entry validation of the restored tree: GPU parity suite, smoke(), default bench line
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01f_gpu_tests.log 2>&1; echo tests=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r01f_smoke.log 2>&1; echo smoke=$?
timeout 600 python bench.py > gpurun_out/r01f_c3.json 2> gpurun_out/r01f_c3.err; echo c3=$?
tail -3 gpurun_out/r01f_gpu_tests.log
