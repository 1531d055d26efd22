# Refresh the range-replay traffic figures for the library that stays in the tree, then one
# bench line to confirm the digest match
set -x
md5sum paper_conf_ipps_qiaoth21_b200/libisp.so
timeout 600 python tools/ncu_traffic.py --tag r03 --out-dir profiles 2>&1 | tail -1
timeout 600 python tools/ncu_traffic.py --tag r03 --workload cfg5 --out-dir profiles 2>&1 | tail -1
cp profiles/r03_traffic_cfg2.json profiles/r03_traffic_cfg5.json gpurun_out/
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r03_bench_final.json 2> gpurun_out/r03_bench_final.err
python -c "
import json
d=json.loads(open('gpurun_out/r03_bench_final.json').read().strip().splitlines()[-1]); r=d['roofline']
print(d['value'], r['frac'], r['duration_us'], r['traffic'], r['traffic_build_matches'], d['clocks'])"
