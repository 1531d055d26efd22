for L in exp_libs/libisp_old.so exp_libs/libisp_tailC.so exp_libs/libisp_tailCm.so; do
  echo "== lib $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_TAIL=0 2>&1 | grep '^{' | cut -c1-100
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" --env ISP_TAIL=0 2>&1 | grep '^{' | cut -c1-100
done
ISP_LIB_PATH=exp_libs/libisp_tailCm.so timeout 600 python -m pytest tests/test_gpu_isp_bodies.py -q -x -k "f32_compiled or separable or strips_isp_f32" 2>&1 | tail -2
