# The remaining r03 profiles re-taken with the in-tree library (counters, paper grid, u8
# family, reference arm), so that every current profile comes from the same file
set -x
md5sum paper_conf_ipps_qiaoth21_b200/libisp.so
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r03_ref.json 2>&1
timeout 600 python tools/bench_u8.py --variant tma --variant warp --variant naive > gpurun_out/r03_u8.jsonl 2>&1
timeout 900 python tools/ncu_counters.py --tag r03 --out-dir gpurun_out > gpurun_out/r03_counters.log 2>&1; tail -1 gpurun_out/r03_counters.log
timeout 1800 python tools/paper_sweep.py > gpurun_out/r03_paper_sweep.json 2> gpurun_out/r03_paper_sweep.err
python -c "
import json
d=json.load(open('gpurun_out/r03_paper_sweep.json')); print(d['auto_matches_best_within_5pct'])"
