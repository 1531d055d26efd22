# Round-3-session measurement of the committed build (one gpurun call).
set -x
md5sum paper_conf_ipps_qiaoth21_b200/libisp.so
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r03_bench.json 2> gpurun_out/r03_bench.err; tail -2 gpurun_out/r03_bench.err
timeout 900 python bench.py --workload cfg5 > gpurun_out/r03_bench_cfg5.json 2> gpurun_out/r03_bench_cfg5.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r03_ref.json 2>&1
timeout 600 python tools/bench_suite.py > gpurun_out/r03_suite.json 2> gpurun_out/r03_suite.err
for m in mirror clamp repeat constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done > gpurun_out/r03_fused.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r03_launches.csv python bench.py --steps 2 --warmup 3 --quick --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_sep_band -s 8 -c 1 -o gpurun_out/r03_sepband python tools/prof_one.py --variant tma --mode clamp --launches 10 > gpurun_out/r03_ncu.log 2>&1
tail -1 gpurun_out/r03_ncu.log
python -c "
import json; d=json.loads(open('gpurun_out/r03_bench.json').read().strip().splitlines()[-1])
print(d['value'], d['roofline'], d['clocks'], d.get('e2e'))"
