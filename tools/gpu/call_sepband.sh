set -x
ISP_F32_BAND=1 timeout 900 python -m pytest tests/test_gpu_isp_bodies.py tests/test_gpu_parity.py -k "f32 or gauss or sep or cfg2 or cfg5" -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -12 | cut -c1-200
timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_F32_BAND=1 --env ISP_F32_BAND=1,ISP_BAND_BANDS=148 --env ISP_F32_BAND=1,ISP_BAND_BANDS=370 2>&1 | grep '^{'
timeout 600 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" --env ISP_F32_BAND=1 2>&1 | grep '^{'
