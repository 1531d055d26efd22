set -x
for gq in 2 1; do ISP_FUSED_G=$gq timeout 900 python -m pytest tests/test_gpu_fused.py -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -3 | cut -c1-200; done
for gq in 2 1; do for m in mirror repeat; do ISP_FUSED_G=$gq timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done; done
