for L in "" exp_libs/libisp_bp.so; do
  echo "== $L"
  ISP_LIB_PATH=$L timeout 600 python tools/bench_knobs.py --cycle --env "" 2>&1 | grep '^{' | cut -c1-100
  ISP_LIB_PATH=$L timeout 600 python bench.py --steps 20 --warmup 5 --quick --no-cpu 2>/dev/null | python -c "
import sys,json; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('bench', d['roofline']['duration_us'], d['roofline']['frac'])"
  ISP_LIB_PATH=$L timeout 600 python bench.py --steps 200 --warmup 5 --quick --no-cpu 2>/dev/null | python -c "
import sys,json; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('bench200', d['roofline']['duration_us'], d['roofline']['frac'])"
done
