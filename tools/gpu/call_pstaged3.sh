set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -x -q -p no:cacheprovider 2>&1 | tail -4
timeout 1200 python tools/bench_knobs.py --cycle --env ISP_TMA_STATIC=1 --env "" \
  --env ISP_P_NWC=4,ISP_P_CTAS=8,ISP_P_RING_KB=24,ISP_P_CH=16 \
  --env ISP_P_NWC=4,ISP_P_CTAS=8,ISP_P_RING_KB=24,ISP_P_CH=32 \
  --env ISP_P_NWC=4,ISP_P_CTAS=8,ISP_P_RING_KB=24,ISP_P_CH=8 \
  --env ISP_P_NWC=4,ISP_P_CTAS=8,ISP_P_RING_KB=16,ISP_P_CH=16 \
  --env ISP_P_NWC=4,ISP_P_CTAS=6,ISP_P_RING_KB=32,ISP_P_CH=16 \
  --env ISP_P_NWC=8,ISP_P_CTAS=4,ISP_P_RING_KB=48,ISP_P_CH=16 \
  --env ISP_P_NWC=8,ISP_P_CTAS=4,ISP_P_RING_KB=48,ISP_P_CH=32 \
  --env ISP_P_NWC=8,ISP_P_CTAS=3,ISP_P_RING_KB=64,ISP_P_CH=32 \
  --env ISP_P_NWC=8,ISP_P_CTAS=2,ISP_P_RING_KB=96,ISP_P_CH=32 \
  --env ISP_P_NWC=12,ISP_P_CTAS=2,ISP_P_RING_KB=96,ISP_P_CH=32 \
  --env ISP_P_NWC=2,ISP_P_CTAS=16,ISP_P_RING_KB=12,ISP_P_CH=16 \
  > gpurun_out/ps3_knobs.jsonl 2>&1
cat gpurun_out/ps3_knobs.jsonl
