set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "band or tile_kernels" -x -q -p no:cacheprovider 2>&1 | tail -3
python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 && \
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_lap_band -s 2 -c 1 -o gpurun_out/r03_lapband2 python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 > gpurun_out/r03_lapband2.log 2>&1
tail -1 gpurun_out/r03_lapband2.log
