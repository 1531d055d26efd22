"""bench.py's multi-rank launch path on CPU (gloo): `bench.py --gpus 2` started without
torchrun re-executes itself under torch.distributed.run with 2 ranks (rendezvous on
127.0.0.1), every rank joins the process group and rank 0 prints one JSON line; a
WORLD_SIZE that disagrees with --gpus is an error, not a silent 1-GPU run."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _json_lines(out):
    return [json.loads(l) for l in out.splitlines() if l.startswith("{")]


@pytest.mark.skipif(sys.platform != "linux", reason="torchrun rendezvous")
def test_gpus2_spawns_two_ranks():
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    env["CUDA_VISIBLE_DEVICES"] = ""          # force the gloo path even on a GPU box
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--check-launch"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1, r.stdout
    d = lines[0]
    assert d["check"] == "launch" and d["world_size"] == 2 and d["ranks_seen"] == 2
    assert d["rank_sum"] == 1 and d["backend"] == "gloo" and d["gpus_requested"] == 2


def test_world_size_mismatch_is_an_error():
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--check-launch"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT, env=env)
    assert r.returncode != 0 and "WORLD_SIZE" in r.stderr


@pytest.mark.gpu
def test_bench_two_ranks_peer_path_one_gpu():
    """bench.py --gpus 2 end to end on a one-GPU box: the test hook ISP_BENCH_SAME_DEVICE=1
    puts both ranks on cuda:0 (gloo process group, CUDA IPC between the processes), so the
    multi-rank code -- handle exchange, peer-direct strip launches, graphs, max-over-ranks
    timing -- runs before a multi-GPU box is available (the numbers are not a measurement)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    env = dict(os.environ, ISP_BENCH_SAME_DEVICE="1")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3",
                        "--quick", "--no-cpu"], capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _json_lines(r.stdout)[-1]
    assert d["n_gpus"] == 2 and d["halo_path"] == "peer" and d["gpu_launches"] == 3 * 4
    assert d["config"]["image"] == [8192, 4096] and d["value"] > 0
