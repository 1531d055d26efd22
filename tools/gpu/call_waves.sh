set -x
for wv in 100 150 185 200 300; do
ISP_BAND_WAVES=$wv timeout 600 python tools/bench_u8.py --only laplace,harris --variant tma 2>&1 | grep '^{'
ISP_BAND_WAVES=$wv timeout 300 python tools/fused_time.py --mode mirror 2>&1 | tail -1
done
timeout 600 python tools/ncu_traffic.py --tag r03 --out-dir gpurun_out 2>&1 | tail -1
timeout 600 python tools/ncu_traffic.py --tag r03 --workload cfg5 --out-dir gpurun_out 2>&1 | tail -1
