set -x
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/membench tools/membench.cu && /tmp/membench 2>&1 | tee gpurun_out/membench.txt | head -40
timeout 900 python tools/bench_knobs.py --cycle --env ISP_TMA_STATIC=1 --env ISP_TMA_STATIC=1,ISP_DEBUG_STAGED=8 \
  --env ISP_TMA_STATIC=1,ISP_DEBUG_STAGED=1 --env ISP_TMA_STATIC=1,ISP_DEBUG_STAGED=2 \
  --env ISP_P_NWC=8,ISP_P_CTAS=4,ISP_P_RING_KB=48 --env ISP_P_NWC=8,ISP_P_CTAS=4,ISP_P_RING_KB=48,ISP_DEBUG_STAGED=8 \
  --env ISP_P_NWC=8,ISP_P_CTAS=1,ISP_P_RING_KB=96,ISP_DEBUG_STAGED=8 \
  > gpurun_out/decomp.jsonl 2>&1
cat gpurun_out/decomp.jsonl
