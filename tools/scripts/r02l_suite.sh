# round 2: peer tier test, then the whole GPU suite
set -x
timeout 600 python -m pytest tests/test_gpu_peer_tier.py -q -m gpu 2>&1 | tail -15
timeout 2400 python -m pytest tests -m gpu -q --durations=10 2>&1 | tail -25
