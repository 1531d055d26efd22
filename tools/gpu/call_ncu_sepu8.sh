# ncu --set full of the u8 Gaussian band kernel (k_sepu8_band) and of the fused kernel on
# the structured cfg3 image path
set -x
timeout 120 python tools/prof_one.py --op gauss_u8 --variant tma --mode mirror --launches 2 && \
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_sepu8_band -s 2 -c 1 -o gpurun_out/r03f_sepu8band python tools/prof_one.py --op gauss_u8 --variant tma --mode mirror --launches 4 > /dev/null 2>&1
ls -la gpurun_out/r03f_sepu8band.ncu-rep
