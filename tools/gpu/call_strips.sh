set -x
timeout 1200 python -m pytest tests/test_gpu_isp_bodies.py tests/test_gpu_parity.py tests/test_gpu_peer_ipc.py -k "strip or peer or shard" -x -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -25 | cut -c1-220
timeout 600 env ISP_BENCH_SAME_DEVICE=1 python -c "print('same-device bench skipped')"
