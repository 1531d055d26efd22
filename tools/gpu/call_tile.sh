timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -q -x -p no:cacheprovider -k "tile or sobel_laplace_harris or harris_threshold" 2>&1 | tail -4
python tools/bench_u8.py --variant tma --variant warp --variant auto 2>&1 | grep '^{' | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['variant'], {k:d[k]['us'] for k in ('sobel','laplace','harris')})"
