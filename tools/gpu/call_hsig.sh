# Harris sign-decision experiment: main lib (HAR_SIGNS=1) vs exp_libs/libisp_hs0.so (per-pair harris2p)
set -x
for L in main hs0; do
  if [ $L = main ]; then unset ISP_LIB_PATH; else export ISP_LIB_PATH=$PWD/exp_libs/libisp_$L.so; fi
  echo "== $L"
  timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider -k "harris or fused or Harris" 2>&1 | tail -2
  for r in 1 2; do timeout 300 python tools/bench_u8.py --variant tma --only harris 2>&1 | tail -1; done
  for m in mirror constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done
done
