set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "band or tile_kernels" -x -q -p no:cacheprovider 2>&1 | tail -3
for L in "" exp_libs/libisp_ld3.so exp_libs/libisp_ld7.so; do
ISP_LIB_PATH=$L timeout 600 python tools/bench_u8.py --only laplace --variant tma --env ISP_BAND_BANDS=148 --env ISP_BAND_BANDS=222 2>&1 | grep '^{'
done
python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 && \
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_lap_band -s 2 -c 1 -o gpurun_out/r03_lapband3 python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 > gpurun_out/r03_lapband3.log 2>&1
