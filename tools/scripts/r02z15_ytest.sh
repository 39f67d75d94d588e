set -x
timeout 900 python -m pytest tests/test_gpu_block.py -q -x -k "grouped or parallel or active_rows" 2>&1 | tail -3
