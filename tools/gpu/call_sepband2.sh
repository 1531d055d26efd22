set -x
for L in "" exp_libs/libisp_sld3.so exp_libs/libisp_sld7.so; do
ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env ISP_F32_BAND=1 --env ISP_F32_BAND=1,ISP_BAND_BANDS=222 --env ISP_F32_BAND=1,ISP_BAND_BANDS=592 2>&1 | grep '^{'
done
ISP_F32_BAND=1 python tools/prof_one.py --variant tma --mode clamp --launches 4 && \
ISP_F32_BAND=1 timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_sep_band -s 2 -c 1 -o gpurun_out/r03_sepband1 python tools/prof_one.py --variant tma --mode clamp --launches 4 > gpurun_out/r03_sepband1.log 2>&1
