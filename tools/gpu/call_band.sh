# Laplace band kernel: parity, then timing against the tile / streaming / naive kernels.
set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "band or tile_kernels" -x -q -p no:cacheprovider 2>&1 | tail -15
timeout 600 python tools/bench_u8.py --only laplace --variant tma --variant warp --variant naive 2>&1 | grep '^{'
timeout 600 python tools/bench_u8.py --only laplace --variant tma --env ISP_BAND_BANDS=148 --env ISP_BAND_BANDS=444 --env ISP_BAND_BANDS=592 --env ISP_BAND_BANDS=888 2>&1 | grep '^{'
for m in clamp repeat constant; do timeout 600 python tools/bench_u8.py --only laplace --mode $m --variant tma 2>&1 | grep '^{'; done
