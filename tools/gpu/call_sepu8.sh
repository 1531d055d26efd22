set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "sepu8 or u8_bodies" -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -15 | cut -c1-200
for nw in 4 2; do ISP_SEPU8_NW=$nw timeout 300 python tools/bench_u8.py --only gauss5 --variant tma 2>&1 | grep '^{'; done
timeout 300 python tools/bench_u8.py --only gauss5 --variant warp --variant naive 2>&1 | grep '^{'
