# Harris strict-bound decision (flat areas decided in f32): full GPU suite + u8 / fused / cfg3 timings
set -x
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -4
timeout 300 python tools/bench_u8.py --variant tma --variant warp 2>&1 | tail -2
for m in mirror constant; do timeout 300 python tools/fused_time.py --mode $m 2>&1 | tail -1; done
timeout 600 python tools/bench_suite.py > gpurun_out/r03h_suite.json 2> gpurun_out/r03h_suite.err
python -c "
import json; d=json.load(open('gpurun_out/r03h_suite.json'))
print(json.dumps(d['cfg3'])[:1500])"
