# Final measurement of the committed build (after the Harris decision change) (one gpurun call); traffic first so that the
# bench lines quote this build's range-replay figure.
set -x
md5sum paper_conf_ipps_qiaoth21_b200/libisp.so
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -4
timeout 600 python tools/ncu_traffic.py --tag r03 --out-dir profiles 2>&1 | tail -1
timeout 600 python tools/ncu_traffic.py --tag r03 --workload cfg5 --out-dir profiles 2>&1 | tail -1
cp profiles/r03_traffic_cfg2.json profiles/r03_traffic_cfg5.json gpurun_out/
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r03_bench.json 2> gpurun_out/r03_bench.err
timeout 900 python bench.py --workload cfg5 --steps 20 --warmup 5 > gpurun_out/r03_bench_cfg5.json 2> gpurun_out/r03_bench_cfg5.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r03_ref.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r03_launches.csv python bench.py --steps 2 --warmup 3 --quick --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_sep_band -s 8 -c 1 -o gpurun_out/r03f_sepband python tools/prof_one.py --variant tma --mode clamp --launches 10 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_har_band -s 2 -c 1 -o gpurun_out/r03f_harband python tools/prof_one.py --op harris --variant tma --mode mirror --launches 4 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_sob_band -s 2 -c 1 -o gpurun_out/r03f_sobband python tools/prof_one.py --op sobel --variant tma --mode mirror --launches 4 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_lap_band -s 2 -c 1 -o gpurun_out/r03f_lapband python tools/prof_one.py --op laplace --variant tma --mode mirror --launches 4 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_fused_band -s 2 -c 1 -o gpurun_out/r03f_fusedband python tools/prof_one.py --op fused3 --variant tma --mode mirror --launches 4 > /dev/null 2>&1
timeout 600 python tools/bench_u8.py --variant tma --variant warp --variant naive > gpurun_out/r03_u8.jsonl 2>&1
for m in mirror clamp repeat constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done > gpurun_out/r03_fused.jsonl
timeout 900 python tools/ncu_counters.py --tag r03 --out-dir gpurun_out > gpurun_out/r03_counters.log 2>&1; tail -1 gpurun_out/r03_counters.log
timeout 1800 python tools/paper_sweep.py > gpurun_out/r03_paper_sweep.json 2> gpurun_out/r03_paper_sweep.err
timeout 600 python tools/bench_suite.py > gpurun_out/r03_suite.json 2> gpurun_out/r03_suite.err
python -c "
import json
for f in ['gpurun_out/r03_bench.json','gpurun_out/r03_bench_cfg5.json']:
    d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, d['value'], d['roofline']['frac'], d['roofline']['duration_us'], d['roofline']['traffic_build_matches'], d['clocks'], d['e2e']['value'])
d=json.load(open('gpurun_out/r03_paper_sweep.json')); print(d['auto_matches_best_within_5pct'])"
