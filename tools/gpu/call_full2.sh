python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -6
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r02b.json 2> gpurun_out/bench_r02b.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_r02b.json').read().strip().splitlines()[-1])
print(d['value'], d['roofline']['frac'], d['roofline']['duration_us'], d['clocks'])"
