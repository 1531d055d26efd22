set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -x -q -p no:cacheprovider 2>&1 | tail -2
timeout 900 python tools/bench_knobs.py --cycle --env "" --env ISP_TAIL=0 > gpurun_out/tail3.jsonl 2>&1
timeout 900 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" --env ISP_TAIL=0 >> gpurun_out/tail3.jsonl 2>&1
cat gpurun_out/tail3.jsonl
python tools/ncu_traffic.py --tag r02b --out-dir gpurun_out 2>&1 | tail -1
