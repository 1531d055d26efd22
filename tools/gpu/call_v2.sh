set -x
for L in main v2; do
  if [ $L = main ]; then unset ISP_LIB_PATH; else export ISP_LIB_PATH=$PWD/exp_libs/libisp_$L.so; fi
  echo "== $L"
  timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider -k "harris or Harris" 2>&1 | tail -1
  for r in 1 2; do timeout 300 python tools/bench_u8.py --variant tma --only harris 2>&1 | tail -1; done
done
