# round 2: configs[1] as one two-level SDXL request step; the Y-mode C3 bench line
set -x
timeout 900 python tools/c2_step.py 10 3 > gpurun_out/r02o_c2.json 2> gpurun_out/r02o_c2.err; tail -3 gpurun_out/r02o_c2.err; head -c 1500 gpurun_out/r02o_c2.json
timeout 900 python bench.py --mode y --no-extras > gpurun_out/r02o_c3_y.json 2> gpurun_out/r02o_c3_y.err; tail -2 gpurun_out/r02o_c3_y.err; head -c 400 gpurun_out/r02o_c3_y.json
