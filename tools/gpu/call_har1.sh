set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "band or tile_kernels or harris" -x -q -p no:cacheprovider 2>&1 | tail -40 | cut -c1-200
timeout 600 python tools/bench_u8.py --only harris,laplace --variant tma --variant warp --env ISP_BAND_BANDS=148 --env ISP_BAND_BANDS=370 2>&1 | grep '^{'
python tools/prof_one.py --op harris --variant tma --mode mirror --launches 4 && \
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_har_band -s 2 -c 1 -o gpurun_out/r03_harband3 python tools/prof_one.py --op harris --variant tma --mode mirror --launches 4 > gpurun_out/r03_harband3.log 2>&1
