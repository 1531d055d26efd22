# Where does the bottom-up band cost come from: memory side (dbg 1: no compute) or compute side?
set -x
for L in "" exp_libs/libisp_old.so; do
  echo "== lib $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --mode clamp --env "" --env ISP_STAGED_REV=0 --env ISP_DEBUG_STAGED=1 --env ISP_DEBUG_STAGED=1,ISP_STAGED_REV=0 --env ISP_DEBUG_STAGED=2 --env ISP_DEBUG_STAGED=2,ISP_STAGED_REV=0 2>&1 | grep '^{'
done
