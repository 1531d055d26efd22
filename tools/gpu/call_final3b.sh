set -x
md5sum paper_conf_ipps_qiaoth21_b200/libisp.so
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r03_bench.json 2> gpurun_out/r03_bench.err
timeout 900 python bench.py --workload cfg5 --steps 20 --warmup 5 > gpurun_out/r03_bench_cfg5.json 2> gpurun_out/r03_bench_cfg5.err
python -c "
import json
for f in ['gpurun_out/r03_bench.json','gpurun_out/r03_bench_cfg5.json']:
    d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, d['value'], d['roofline']['frac'], d['roofline']['duration_us'], d['clocks'])"
