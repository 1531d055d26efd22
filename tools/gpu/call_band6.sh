set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "band or tile_kernels" -x -q -p no:cacheprovider 2>&1 | grep -v "^E  *[|^$" | tail -40
timeout 600 python tools/bench_u8.py --only laplace --variant tma --env ISP_BAND_BANDS=148 --env ISP_BAND_BANDS=185 --env ISP_BAND_BANDS=296 --env ISP_BAND_NW=2 --env ISP_BAND_NW=2,ISP_BAND_BANDS=148 2>&1 | grep '^{'
python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 && \
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_lap_band -s 2 -c 1 -o gpurun_out/r03_lapband6 python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 > gpurun_out/r03_lapband6.log 2>&1
