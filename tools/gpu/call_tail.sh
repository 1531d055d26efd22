set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -x -q -p no:cacheprovider 2>&1 | tail -4
timeout 900 python tools/bench_knobs.py --cycle --env "" --env ISP_TAIL=0 --env ISP_TAIL=1,ISP_STAGES=6 --env ISP_TAIL=1,ISP_STAGES=3 \
  --env ISP_TMA_PERSIST=1 > gpurun_out/tail.jsonl 2>&1
cat gpurun_out/tail.jsonl
for m in clamp mirror repeat constant; do timeout 300 python tools/bench_knobs.py --mode $m --env "" --env ISP_TAIL=0 ; done 2>&1 | tee gpurun_out/tail_modes.jsonl
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_staged -s 3 -c 4 python tools/prof_one.py --variant tma --mode clamp --launches 6 2>&1 | grep -E "dram__|gpu__time" | head -12
