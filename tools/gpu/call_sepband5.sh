set -x
timeout 600 python -m pytest tests/test_gpu_isp_bodies.py -k "sep_band" -x -q -p no:cacheprovider 2>&1 | tail -2
for L in "" exp_libs/libisp_m8.so exp_libs/libisp_d4.so; do
ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_BAND_BANDS=259 --env ISP_BAND_BANDS=296 --env ISP_BAND_BANDS=148 2>&1 | grep '^{'
ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" --env ISP_BAND_BANDS=108 2>&1 | grep '^{'
done
