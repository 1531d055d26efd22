set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -x -q -p no:cacheprovider 2>&1 | tail -2
timeout 900 python tools/bench_knobs.py --cycle --env "" --env ISP_TAIL=0 --env ISP_STAGES=3 --env ISP_STAGES=5 --env ISP_EDGE_W=128 --env ISP_EDGE_W=0 > gpurun_out/tail2.jsonl 2>&1
cat gpurun_out/tail2.jsonl
timeout 900 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" --env ISP_TAIL=0 2>&1 | tee gpurun_out/tail2_cfg5.jsonl
python tools/ncu_traffic.py --tag r02a --out-dir gpurun_out 2>&1 | tail -2
