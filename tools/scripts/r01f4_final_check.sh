# final code of the round: full GPU suite, smoke, default bench line
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01f4_gpu_tests.log 2>&1; echo tests=$?
tail -3 gpurun_out/r01f4_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01f4_smoke.log 2>&1; echo smoke=$?
tail -1 gpurun_out/r01f4_smoke.log
timeout 600 python bench.py > gpurun_out/r01f4_c3.json 2> gpurun_out/r01f4_c3.err; echo c3=$?
