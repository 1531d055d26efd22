set -x
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/full_tests.log
tail -15 gpurun_out/full_tests.log
timeout 900 python tools/ncu_counters.py --tag r02 --out-dir gpurun_out 2>&1 | tail -3
timeout 600 python tools/ncu_traffic.py --tag r02 --out-dir gpurun_out 2>&1 | tail -1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r02a.json 2> gpurun_out/bench_r02a.err
tail -c 600 gpurun_out/bench_r02a.json
