# round 2: where the step's time beyond the serialised kernel sum goes -- PDL on / off, k = 37
set -x
timeout 900 python tools/step_probe.py C3 2 37 6 > gpurun_out/r02g_pdl.jsonl 2>/dev/null; cat gpurun_out/r02g_pdl.jsonl
FPS_KERNEL_FLAGS=64 timeout 900 python tools/step_probe.py C3 2 37 6 > gpurun_out/r02g_nopdl.jsonl 2>/dev/null; cat gpurun_out/r02g_nopdl.jsonl
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv
