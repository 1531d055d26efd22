for L in "" exp_libs/libisp_pf1.so exp_libs/libisp_px8pf1.so; do
  ISP_LIB_PATH=$L timeout 300 python tools/bench_u8.py --variant warp --variant tma --variant naive 2>&1 | grep '^{' | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['px_u8'] or 'base', d['variant'], {k:d[k]['us'] for k in ('sobel','laplace','harris')})"
done
