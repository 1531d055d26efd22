"""Peer-direct strips across PROCESSES: P worker processes, one rank
each, all on cuda:0 (every gpurun call has one GPU; CUDA IPC between processes on one
device is the same mechanism as between GPUs over NVLink).  Each rank owns only its strip;
the 72-byte IPC handles are exchanged over a gloo process group, isp_shard_peer_attach maps
the neighbours (ring neighbours for Repeat; P = 2 maps one strip for both sides), and ONE
launch per rank reads the neighbour rows straight from the other processes' memory.  The
gathered strips equal the single-image result bitwise, every border mode."""
import os
import tempfile

import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu

MODES = ["clamp", "mirror", "repeat", "constant"]
H, W = 203, 2052


def _mask(m):
    return np.random.default_rng(m).random((m, m)).astype(np.float32)


def _worker(rank, nranks, port, outdir, m):
    import torch.distributed as dist

    import paper_conf_ipps_qiaoth21_b200 as isp
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=nranks)
    torch.cuda.set_device(0)
    img = synth.uniform_f32(H, W, 81)
    y0, sh = isp.isp_shard_rows(H, rank, nranks)
    strip = torch.from_numpy(np.ascontiguousarray(img[y0:y0 + sh])).cuda()
    torch.cuda.synchronize()
    handles = [None] * nranks
    dist.all_gather_object(handles, isp.isp_shard_peer_handle(strip))
    pp = isp.isp_shard_peer_attach(rank, nranks, strip, handles, ring=True)
    dist.barrier()                 # every strip holds its data before any rank reads it
    for mode in MODES:
        for v in ["tma", "warp", "naive"]:
            out = isp.isp_shard_peer_filter_f32(pp, H, _mask(m), mode, 0.25, variant=v)
            torch.cuda.synchronize()
            np.save(os.path.join(outdir, f"{mode}_{v}_{rank}.npy"), out.cpu().numpy())
    dist.barrier()                 # no rank unmaps / frees while a neighbour still reads
    isp.isp_shard_peer_close(pp)
    dist.destroy_process_group()


@pytest.mark.parametrize("nranks", [2, 3])
@pytest.mark.parametrize("m", [5, 7])
def test_peer_strips_across_processes(nranks, m):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import socket

    import torch.multiprocessing as mp

    import paper_conf_ipps_qiaoth21_b200 as isp
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    with tempfile.TemporaryDirectory() as outdir:
        mp.spawn(_worker, args=(nranks, port, outdir, m), nprocs=nranks, join=True)
        full = torch.from_numpy(synth.uniform_f32(H, W, 81)).cuda()
        for mode in MODES:
            for v in ["tma", "warp", "naive"]:
                ref = isp.isp_filter_ex(full, _mask(m), mode, 0.25, variant=v).cpu().numpy()
                got = np.concatenate([np.load(os.path.join(outdir, f"{mode}_{v}_{r}.npy")) for r in range(nranks)])
                np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} P={nranks} m={m}")
