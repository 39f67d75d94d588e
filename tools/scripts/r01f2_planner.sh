# after the planner prices the transition block: full GPU suite, smoke, bench lines of the configs
# whose plan can move (C3 default, C4, C2A, C2B)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01f2_gpu_tests.log 2>&1; echo tests=$?
tail -3 gpurun_out/r01f2_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01f2_smoke.log 2>&1; echo smoke=$?
timeout 600 python bench.py > gpurun_out/r01f2_c3.json 2> gpurun_out/r01f2_c3.err; echo c3=$?
timeout 900 python bench.py --config C4 --no-cpu > gpurun_out/r01f2_c4.json 2> gpurun_out/r01f2_c4.err; echo c4=$?
timeout 400 python bench.py --config C2A --no-cpu > gpurun_out/r01f2_c2a.json 2> gpurun_out/r01f2_c2a.err; echo c2a=$?
timeout 600 python bench.py --config C2B --no-cpu > gpurun_out/r01f2_c2b.json 2> gpurun_out/r01f2_c2b.err; echo c2b=$?
