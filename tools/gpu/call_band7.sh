set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "band or tile_kernels" -x -q -p no:cacheprovider 2>&1 | tail -60 | cut -c1-200
