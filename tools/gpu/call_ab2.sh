for L in exp_libs/libisp_old640.so exp_libs/libisp_new512.so; do
  echo "== lib $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_TAIL=0 2>&1 | grep '^{' | cut -c1-120
done
