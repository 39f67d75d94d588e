# round 2: TMA row gather with eager stores -- correctness, isolated rate per CTA count, C3 sweep
set -x
timeout 600 python -m pytest tests/test_gpu_rows.py tests/test_gpu_engine.py -q -x -k "prefetch or copy_methods or delayed or cross_step" 2>&1 | tail -3
for c in 2 4; do
PROBE_CTAS=$c timeout 900 python tools/step_probe.py C3 3 36,38,40,42 6 > gpurun_out/r02e_m3c$c.jsonl 2> gpurun_out/r02e_m3c$c.err
cat gpurun_out/r02e_m3c$c.jsonl
done
