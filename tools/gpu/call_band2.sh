set -x
for L in "" exp_libs/libisp_ld8.so exp_libs/libisp_ld12.so; do
ISP_LIB_PATH=$L timeout 600 python tools/bench_u8.py --only laplace,copy --variant tma --env ISP_BAND_BANDS=148 --env ISP_BAND_BANDS=222 2>&1 | grep '^{'
done
