# round 2: step probe at C3 -- loads vs no-load arm per H2D method and plan; SM reservation A/B
set -x
timeout 900 python tools/step_probe.py C3 3,2 38,40,42 6 > gpurun_out/r02b_probe.jsonl 2> gpurun_out/r02b_probe.err
FPS_SM_RESERVE=0 timeout 600 python tools/step_probe.py C3 3 40 6 > gpurun_out/r02b_probe_res0.jsonl 2> gpurun_out/r02b_probe_res0.err
cat gpurun_out/r02b_probe.jsonl gpurun_out/r02b_probe_res0.jsonl
tail -3 gpurun_out/r02b_probe.err
