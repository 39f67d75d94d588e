# TMA row gather (method 3) in the step: does it lose its reserved SMs to early-launched (PDL)
# compute CTAs?  C3 probe: default, high-priority load stream, PDL off
set -x
timeout 900 python tools/step_probe.py C3 3,2 40,42,44 6 > gpurun_out/r02z4_default.jsonl 2> gpurun_out/r02z4_default.err
PROBE_LOAD_PRIO=-5 timeout 900 python tools/step_probe.py C3 3 40,42,44 6 > gpurun_out/r02z4_prio.jsonl 2> gpurun_out/r02z4_prio.err
FPS_KERNEL_FLAGS=64 timeout 900 python tools/step_probe.py C3 3,2 40,42,44 6 > gpurun_out/r02z4_nopdl.jsonl 2> gpurun_out/r02z4_nopdl.err
FPS_KERNEL_FLAGS=64 PROBE_LOAD_PRIO=-5 timeout 900 python tools/step_probe.py C3 3 40,42,44 6 > gpurun_out/r02z4_nopdl_prio.jsonl 2> gpurun_out/r02z4_nopdl_prio.err
tail -3 gpurun_out/r02z4_*.err
cat gpurun_out/r02z4_*.jsonl
