timeout 900 python -m pytest tests/test_gpu_fused.py -q -x -p no:cacheprovider 2>&1 | tail -4
python tools/fused_time.py
for m in clamp repeat constant; do python tools/fused_time.py --mode $m; done
