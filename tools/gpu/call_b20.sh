for i in 1 2 3; do timeout 300 python bench.py --steps 20 --warmup 5 --quick 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('k20', d['value'], round(d['roofline']['duration_us'],2), round(d['roofline']['frac'],3), d['clocks'])"; done
timeout 300 python bench.py --quick 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('k200', d['value'], round(d['roofline']['duration_us'],2), round(d['roofline']['frac'],3), d['clocks'])"
timeout 300 python bench.py --workload cfg5 --steps 20 --warmup 5 --quick 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('cfg5 k20', d['value'], round(d['roofline']['duration_us'],2), round(d['roofline']['frac'],3), d['clocks'])"
