# HEAD check after the CTA-pair GEMM change: GPU suite, smoke, default bench line, Y-mode line
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -6
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1500 python bench.py > gpurun_out/r02z3_c3.json 2> gpurun_out/r02z3_c3.err; tail -3 gpurun_out/r02z3_c3.err
timeout 1500 python bench.py --mode y --no-cpu > gpurun_out/r02z3_c3_y.json 2> gpurun_out/r02z3_c3_y.err; tail -3 gpurun_out/r02z3_c3_y.err
