set -x
ISP_FUSED_SPLIT=1 timeout 900 python -m pytest tests/test_gpu_fused.py -x -q -p no:cacheprovider 2>&1 | tail -2
for m in mirror repeat; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; ISP_FUSED_SPLIT=1 timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done
timeout 1500 python -m pytest tests/test_gpu_parity.py -k cfg5 -x -q -p no:cacheprovider 2>&1 | tail -2
