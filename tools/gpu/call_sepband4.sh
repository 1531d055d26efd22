set -x
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -15 | cut -c1-200
timeout 900 python bench.py --steps 2000 --warmup 20 > gpurun_out/r03_bench_try.json 2> gpurun_out/r03_bench_try.err; tail -c 600 gpurun_out/r03_bench_try.json
timeout 900 python bench.py --workload cfg5 --steps 200 --warmup 5 > gpurun_out/r03_bench_cfg5_try.json 2>&1; tail -c 300 gpurun_out/r03_bench_cfg5_try.json
