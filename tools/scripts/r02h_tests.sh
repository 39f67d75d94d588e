# round 2: the new GPU tests only (full-scale parity, flow-blend sampler, record)
set -x
timeout 2400 python -m pytest tests/test_gpu_fullscale.py tests/test_gpu_engine.py -m gpu -q --durations=8 -k "fullscale or flow_blend or record or flux" 2>&1 | tail -30
