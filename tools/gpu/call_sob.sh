set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "sobel" -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -15 | cut -c1-200
timeout 600 python tools/bench_u8.py --variant tma --variant warp --variant auto 2>&1 | grep '^{'
for m in mirror clamp; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done
