set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py tests/test_gpu_parity.py -k "harris" -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -15 | cut -c1-200
for gq in 2 1; do ISP_HARRIS_G=$gq timeout 300 python tools/bench_u8.py --only harris --variant tma 2>&1 | grep '^{'; done
for wv in 150 200; do ISP_BAND_WAVES=$wv timeout 300 python tools/bench_u8.py --only harris --variant tma 2>&1 | grep '^{'; done
