set -x
timeout 900 python -m pytest tests/test_gpu_fused.py -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -30 | cut -c1-220
for m in mirror clamp repeat constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done
python tools/prof_one.py --op fused3 --variant tma --mode mirror --launches 4 && \
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_fused_band -s 2 -c 1 -o gpurun_out/r03_fusedband3 python tools/prof_one.py --op fused3 --variant tma --mode mirror --launches 4 > gpurun_out/r03_fusedband3.log 2>&1
timeout 600 python tools/bench_u8.py --only harris,laplace --variant tma 2>&1 | grep '^{'
