for L in "" exp_libs/libisp_th32.so exp_libs/libisp_th16.so; do
ISP_LIB_PATH=$L python tools/bench_u8.py --variant tma 2>&1 | grep '^{' | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('$L', d['variant'], {k:d[k]['us'] for k in ('laplace','harris')})"
done
