# round 2: C3 plan sweep per H2D method; TMA gather on 2 vs 4 CTAs (variable ring depth)
set -x
PROBE_CTAS=2 timeout 900 python tools/step_probe.py C3 3 35,36,37,38,39,40 6 > gpurun_out/r02d_m3c2.jsonl 2> gpurun_out/r02d_m3c2.err
PROBE_CTAS=4 timeout 900 python tools/step_probe.py C3 3 35,36,37,38,39 6 > gpurun_out/r02d_m3c4.jsonl 2> gpurun_out/r02d_m3c4.err
timeout 900 python tools/step_probe.py C3 2 34,35,36,37,38 6 > gpurun_out/r02d_m2.jsonl 2> gpurun_out/r02d_m2.err
PROBE_MODE=y PROBE_CTAS=2 timeout 900 python tools/step_probe.py C3 3,2 50,54,57 6 > gpurun_out/r02d_y.jsonl 2> gpurun_out/r02d_y.err
cat gpurun_out/r02d_*.jsonl
tail -2 gpurun_out/r02d_*.err
