set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "band or tile_kernels" -x -q -p no:cacheprovider 2>&1 | tail -15
timeout 600 python tools/bench_u8.py --only laplace,copy --variant tma --env ISP_BAND_BANDS=148 --env ISP_BAND_BANDS=222 2>&1 | grep '^{'
for m in clamp repeat constant; do timeout 600 python tools/bench_u8.py --only laplace --mode $m --variant tma 2>&1 | grep '^{'; done
