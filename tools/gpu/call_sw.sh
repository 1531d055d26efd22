for L in "" exp_libs/libisp_sw2.so exp_libs/libisp_sw8.so; do
  echo "== $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_STAGES=6 --env ISP_STAGES=3 2>&1 | grep '^{' | cut -c1-110
done
