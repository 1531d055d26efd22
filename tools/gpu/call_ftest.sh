set -x
timeout 900 python -m pytest tests/test_gpu_fused.py -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -25 | cut -c1-220
