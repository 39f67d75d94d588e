# per-run DMA (method 1) in the C3 step vs whole-entry DMA: loaded vs no-load at fixed plans
set -x
timeout 900 python tools/step_probe.py C3 1,2 36,38,40,42 6 > gpurun_out/r02z11_m1.jsonl 2> gpurun_out/r02z11_m1.err
cat gpurun_out/r02z11_m1.jsonl
