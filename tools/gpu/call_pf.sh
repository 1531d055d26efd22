for L in exp_libs/libisp_base.so exp_libs/libisp_pf.so; do
  echo "== $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_TAIL_L2=0 2>&1 | grep '^{' | cut -c1-100
  ISP_LIB_PATH=$L timeout 600 python bench.py --steps 20 --warmup 5 --quick --no-cpu 2>/dev/null | python -c "
import sys,json; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('bench', d['roofline']['duration_us'], d['roofline']['frac'])"
done
ISP_LIB_PATH=exp_libs/libisp_pf.so timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_staged -s 8 -c 4 python tools/prof_one.py --variant tma --mode clamp --launches 12 2>&1 | grep -E "dram__bytes_read|gpu__time"
