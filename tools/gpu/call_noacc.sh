# fused band kernel: Harris running pair (main) vs the three-row ring (noacc), strict decision in both
set -x
for L in main noacc; do
  if [ $L = main ]; then unset ISP_LIB_PATH; else export ISP_LIB_PATH=$PWD/exp_libs/libisp_$L.so; fi
  echo "== $L"
  timeout 600 python -m pytest tests/test_gpu_fused.py -q -p no:cacheprovider 2>&1 | tail -1
  for m in mirror constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done
done
