"""Multi-GPU row-strip path on CPU: world_size 2 / 3 with the gloo backend.

Each rank takes the schedule the library computes (isp_shard_schedule, pure host code
in libisp.so), executes its point-to-point ops in order with torch.distributed
isend/irecv on CPU tensors (standing in for ncclSend/ncclRecv inside one group), then
evaluates each launch of the schedule with the CPU oracle on the rows it may read
(t_real / b_real: image border vs halo rows).  The stitched strips must equal the
unsharded oracle -- for every border mode, including the Repeat ring wrap."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

MODES = ["clamp", "mirror", "repeat", "constant"]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, H, W, m, result_q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    import paper_conf_ipps_qiaoth21_b200 as isp
    import synth

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    img = synth.uniform_f32(H, W, 42)                   # every rank can generate the seeded input
    mask = np.random.default_rng(m).random((m, m)).astype(np.float32)
    hy, halo = m // 2, m // 2 + 1
    out = {}
    for mode in MODES:
        sc = isp.isp_shard_schedule(H, rank, world, halo, hy, mode)
        y0, sh = sc["y0"], sc["strip_h"]
        buf = np.full((sh + 2 * halo, W), np.nan, dtype=np.float32)
        buf[halo:halo + sh] = img[y0:y0 + sh]            # own rows only; halos must arrive
        reqs, tensors = [], []
        for kind, peer, row, n in sc["ops"]:
            t = torch.from_numpy(np.ascontiguousarray(buf[row:row + n])) if kind == 0 else torch.empty((n, W))
            tensors.append((kind, row, n, t))
            reqs.append(dist.isend(t, peer) if kind == 0 else dist.irecv(t, peer))
        for r in reqs:
            r.wait()
        for kind, row, n, t in tensors:
            if kind == 1:
                buf[row:row + n] = t.numpy()
        res = np.full((sh, W), np.nan)
        for (oy0, n, ylim, t_real, b_real, after) in sc["launch"]:
            if n <= 0:
                continue
            lo = 0 if t_real else oy0 - hy
            hi = H if b_real else oy0 + n + hy
            assert hi <= ylim, "launch reads past its resident rows"
            sub = buf[lo - y0 + halo: hi - y0 + halo]
            assert not np.isnan(sub).any(), f"rank {rank} {mode}: launch reads rows not yet received"
            r = oracle.filter_f64(sub, mask, mode, 0.25, rows=(oy0 - lo, oy0 - lo + n))
            res[oy0 - y0: oy0 - y0 + n] = r
        out[mode] = (y0, res)
    result_q.put((rank, out))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,H,m", [(2, 40, 5), (2, 23, 7), (3, 61, 3), (3, 30, 9)])
def test_row_strips_gloo(world, H, m):
    import oracle
    import paper_conf_ipps_qiaoth21_b200 as isp
    import synth
    isp.lib()
    oracle.build_oracle()
    W = 37
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, H, W, m, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    img = synth.uniform_f32(H, W, 42)
    mask = np.random.default_rng(m).random((m, m)).astype(np.float32)
    for mode in MODES:
        ref = oracle.filter_f64(img, mask, mode, 0.25)
        got = np.full((H, W), np.nan)
        for r in range(world):
            y0, res = results[r][mode]
            got[y0:y0 + res.shape[0]] = res
        np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12, err_msg=mode)
