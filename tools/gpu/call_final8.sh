# Final measurement (fused: single Harris vote, dx / dy outputs as a template parameter): GPU suite, traffic of the
# in-tree library, bench lines, fused / u8 timings, the fused ncu capture
set -x
md5sum paper_conf_ipps_qiaoth21_b200/libisp.so
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -3
timeout 600 python tools/ncu_traffic.py --tag r03 --out-dir profiles 2>&1 | tail -1
timeout 600 python tools/ncu_traffic.py --tag r03 --workload cfg5 --out-dir profiles 2>&1 | tail -1
cp profiles/r03_traffic_cfg2.json profiles/r03_traffic_cfg5.json gpurun_out/
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r03_bench.json 2> gpurun_out/r03_bench.err
timeout 900 python bench.py --workload cfg5 --steps 20 --warmup 5 > gpurun_out/r03_bench_cfg5.json 2> gpurun_out/r03_bench_cfg5.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r03_launches.csv python bench.py --steps 2 --warmup 3 --quick --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_fused_band -s 2 -c 1 -o gpurun_out/r03f_fusedband python tools/prof_one.py --op fused3 --variant tma --mode mirror --launches 4 > /dev/null 2>&1
for m in mirror clamp repeat constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done > gpurun_out/r03_fused.jsonl
timeout 600 python tools/bench_suite.py > gpurun_out/r03_suite.json 2> gpurun_out/r03_suite.err
python -c "
import json
for f in ['gpurun_out/r03_bench.json','gpurun_out/r03_bench_cfg5.json']:
    d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, d['value'], d['roofline']['frac'], d['roofline']['duration_us'], d['roofline']['traffic_build_matches'], d['clocks'], d['e2e']['value'])
"
cat gpurun_out/r03_fused.jsonl
