timeout 600 python -m pytest tests/test_gpu_isp_bodies.py -k "harris" -x -q -p no:cacheprovider 2>&1 | tail -2
for L in "" exp_libs/libisp_hold.so; do ISP_LIB_PATH=$L timeout 300 python tools/bench_u8.py --only harris --variant tma 2>&1 | grep '^{'; done
