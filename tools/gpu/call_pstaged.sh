# persistent staged kernel: parity of the TMA bodies + knob sweep on cfg2
set -x
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -x -q -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/ps_tests.log
tail -15 gpurun_out/ps_tests.log
timeout 900 python tools/bench_knobs.py --cycle --env "" --env ISP_TMA_STATIC=1 --env ISP_P_CH=8 --env ISP_P_CH=32 \
  --env ISP_P_CH=64 --env ISP_P_NWC=4 --env ISP_P_NWC=16 --env ISP_P_CTAS=2,ISP_P_RING_KB=96 \
  --env ISP_P_CTAS=2,ISP_P_RING_KB=48 --env ISP_P_RING_KB=48 --env ISP_P_RING_KB=160 \
  --env ISP_P_NWC=4,ISP_P_CTAS=2,ISP_P_RING_KB=64 --env ISP_P_NWC=4,ISP_P_CTAS=4,ISP_P_RING_KB=40 \
  > gpurun_out/ps_knobs.jsonl 2>&1
cat gpurun_out/ps_knobs.jsonl
for m in clamp mirror repeat constant; do timeout 300 python tools/bench_knobs.py --mode $m --env "" --env ISP_TMA_STATIC=1 ; done 2>&1 | tee gpurun_out/ps_modes.jsonl
