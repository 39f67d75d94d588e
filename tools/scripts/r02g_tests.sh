# round 2: full GPU suite incl. the new full-scale parity tests, flow-blend sampler, record
set -x
timeout 2400 python -m pytest tests -m gpu -q -x --durations=15 2>&1 | tail -40
