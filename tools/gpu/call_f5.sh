for L in "" exp_libs/libisp_f5.so; do ISP_LIB_PATH=$L timeout 300 python tools/fused_time.py --mode mirror 2>&1 | tail -1; done
