timeout 900 python -m pytest tests/test_gpu_peer_ipc.py -q -x -p no:cacheprovider 2>&1 | tail -15
