# Harris / fused accumulator-state experiment: main lib + two variant builds (exp_libs/)
set -x
for L in main hA hB; do
  if [ $L = main ]; then unset ISP_LIB_PATH; else export ISP_LIB_PATH=$PWD/exp_libs/libisp_$L.so; fi
  echo "== $L"
  timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider -k "harris or fused or Harris" 2>&1 | tail -2
  timeout 300 python tools/bench_u8.py --variant tma --only harris 2>&1 | tail -1
  for m in mirror constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done
done
