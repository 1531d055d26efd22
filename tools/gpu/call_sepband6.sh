set -x
for rep in 1 2; do
for L in "" exp_libs/libisp_l128.so exp_libs/libisp_m8.so; do
ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env ISP_BAND_BANDS=222 --env ISP_BAND_BANDS=240 --env ISP_BAND_BANDS=259 --env ISP_BAND_BANDS=280 2>&1 | grep '^{'
done
done
