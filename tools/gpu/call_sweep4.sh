set -x
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
ISP_LIB_PATH=exp_libs/libisp_h6.so timeout 600 python tools/bench_u8.py --only harris --variant tma 2>&1 | grep '^{'
timeout 600 python tools/bench_u8.py --only harris --variant tma 2>&1 | grep '^{'
bash tools/gpu/call_sweep3.sh
