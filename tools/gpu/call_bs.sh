for K in 20 20 200; do
  timeout 600 python bench.py --steps $K --warmup 5 --quick --no-cpu 2>/dev/null | python -c "
import sys,json; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('bench K=$K', d['roofline']['duration_us'], d['roofline']['frac'], d['value'])"
done
