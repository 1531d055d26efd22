ISP_TAIL=0 timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_staged -s 3 -c 1 -o gpurun_out/ab_new python tools/prof_one.py --variant tma --mode clamp --launches 4 > /dev/null 2>&1
ISP_TAIL=0 ISP_LIB_PATH=exp_libs/libisp_old640.so timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_staged -s 3 -c 1 -o gpurun_out/ab_old python tools/prof_one.py --variant tma --mode clamp --launches 4 > /dev/null 2>&1
ls gpurun_out
