set -x
timeout 900 python -m pytest tests/test_gpu_rows.py -q -x 2>&1 | tail -2
