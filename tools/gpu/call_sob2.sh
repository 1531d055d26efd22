set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py tests/test_gpu_parity.py -k "sobel" -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -15 | cut -c1-200
for gq in 2 1; do ISP_SOBEL_G=$gq timeout 300 python tools/bench_u8.py --only sobel --variant tma 2>&1 | grep '^{'; done
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
