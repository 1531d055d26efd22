set -x
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_isp_bodies.py -k "sepu8 or sep_band" -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -20 | cut -c1-200
bash tools/gpu/call_sweep3.sh
