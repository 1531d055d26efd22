timeout 900 python -m pytest tests/test_gpu_ablations.py tests/test_gpu_isp_bodies.py -q -x -p no:cacheprovider -k "tex or peer or split" 2>&1 | tail -25
