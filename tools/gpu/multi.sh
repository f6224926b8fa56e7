set -x
timeout 1200 python -m pytest tests/test_multigpu.py -x -q -m gpu 2>&1 | tail -15
