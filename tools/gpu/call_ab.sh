set -x
for L in "" exp_libs/libisp_old.so exp_libs/libisp_nominb.so; do
  echo "== lib $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_TAIL=0 2>&1 | grep '^{'
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" 2>&1 | grep '^{'
done
