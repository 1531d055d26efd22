ISP_BENCH_SAME_DEVICE=1 timeout 600 python bench.py --gpus 2 --steps 5 --warmup 3 --quick --no-cpu > gpurun_out/mr2.log 2>&1; tail -c 1500 gpurun_out/mr2.log
ISP_BENCH_SAME_DEVICE=1 timeout 600 python bench.py --gpus 3 --steps 5 --warmup 3 --quick --no-cpu --workload cfg5 > gpurun_out/mr3.log 2>&1; tail -c 1500 gpurun_out/mr3.log
