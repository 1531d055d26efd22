set -x
for L in exp_libs/libisp_sld2.so exp_libs/libisp_sld3.so exp_libs/libisp_sld4.so; do
ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env ISP_F32_BAND=1,ISP_BAND_BANDS=185 --env ISP_F32_BAND=1,ISP_BAND_BANDS=222 --env ISP_F32_BAND=1,ISP_BAND_BANDS=259 --env ISP_F32_BAND=1,ISP_BAND_BANDS=296 --env ISP_F32_BAND=1,ISP_BAND_BANDS=333 2>&1 | grep '^{'
ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env ISP_F32_BAND=1 --env ISP_F32_BAND=1,ISP_BAND_BANDS=54 --env ISP_F32_BAND=1,ISP_BAND_BANDS=81 --env ISP_F32_BAND=1,ISP_BAND_BANDS=108 2>&1 | grep '^{'
done
