# round 2: §6.6 overheads on the real engine (NEXT-3)
set -x
timeout 900 python tools/overheads.py > gpurun_out/r02k_overheads.json 2> gpurun_out/r02k_overheads.err; tail -3 gpurun_out/r02k_overheads.err; cat gpurun_out/r02k_overheads.json
