set -x
python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 && \
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_lap_band -s 2 -c 1 -o gpurun_out/r03_lapband python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 > gpurun_out/r03_lapband.log 2>&1
tail -3 gpurun_out/r03_lapband.log
