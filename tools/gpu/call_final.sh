# Round-2 final measurement of the committed build (one gpurun call).
set -x
md5sum paper_conf_ipps_qiaoth21_b200/libisp.so
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -4
timeout 600 python tools/ncu_traffic.py --tag r02 --out-dir gpurun_out 2>&1 | tail -2
timeout 600 python tools/ncu_traffic.py --tag r02 --workload cfg5 --out-dir gpurun_out 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err; tail -2 gpurun_out/r02_bench.err
timeout 900 python bench.py --workload cfg5 > gpurun_out/r02_bench_cfg5.json 2> gpurun_out/r02_bench_cfg5.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02_ref.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02_launches.csv python bench.py --steps 2 --warmup 3 --quick --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_staged -s 8 -c 1 -o gpurun_out/r02_staged python tools/prof_one.py --variant tma --mode clamp --launches 10 > gpurun_out/r02_ncu.log 2>&1
tail -2 gpurun_out/r02_ncu.log
python -c "
import json; d=json.loads(open('gpurun_out/r02_bench.json').read().strip().splitlines()[-1])
print(d['value'], d['roofline'], d['clocks'], d.get('e2e'))"
