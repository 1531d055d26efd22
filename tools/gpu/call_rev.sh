# A/B of the alternating band direction (Geom::rev) on the cfg2 / cfg5 staged kernels.
set -x
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider 2>&1 | tail -5
for L in "" exp_libs/libisp_old.so; do
  echo "== lib $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_STAGED_REV=0 --env ISP_STAGES=4 2>&1 | grep '^{'
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" --env ISP_STAGED_REV=0 2>&1 | grep '^{'
done
timeout 600 python tools/ncu_traffic.py --tag r03 --out-dir gpurun_out 2>&1 | tail -2
ISP_STAGED_REV=0 timeout 600 python tools/ncu_traffic.py --tag r03norev --out-dir gpurun_out 2>&1 | tail -2
