#!/usr/bin/env python
"""Time the fused cfg3 pipeline (isp_pipeline_cfg3_u8) vs the three launches on 4096^2 u8,
Mirror, CUDA graph of 12 launches over rotating buffers (tools/bench_suite.time_launch).
    python tools/fused_time.py [--size 4096] [--mode mirror]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import torch  # noqa: E402

import paper_conf_ipps_qiaoth21_b200 as isp  # noqa: E402
import synth  # noqa: E402
from bench_suite import time_launch  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--size", type=int, default=4096)
    ap.add_argument("--mode", default="mirror")
    a = ap.parse_args()
    n, nb = a.size, 6
    imgs = [torch.from_numpy(synth.structured_u8(n, n, 3 + i)).cuda() for i in range(nb)]
    outs = [[torch.empty_like(imgs[0]) for _ in range(3)] for _ in range(nb)]
    dxs = [torch.empty((n, n), dtype=torch.int16, device="cuda") for _ in range(nb)]
    dys = [torch.empty_like(d) for d in dxs]
    res = {"size": n, "mode": a.mode, "env_v1": bool(os.environ.get("ISP_FUSED_V1"))}
    for v in ["auto", "warp", "naive"]:   # band kernel, tile-ISP kernel, general kernel
        us, _ = time_launch(lambda i: isp.isp_pipeline_cfg3_u8(imgs[i % nb], a.mode, mag=outs[i % nb][0],
                                                               lap=outs[i % nb][1], harris=outs[i % nb][2],
                                                               variant=v), nb)
        res[f"fused_{v}_us"] = round(us, 2)

    def three(i):
        k = i % nb
        isp.isp_sobel_u8(imgs[k], a.mode, dx=dxs[k], dy=dys[k], mag=outs[k][0])
        isp.isp_laplace5_u8(imgs[k], a.mode, out=outs[k][1])
        isp.isp_harris_u8(dxs[k], dys[k], a.mode, out=outs[k][2])
    us, _ = time_launch(three, nb)
    res["three_launches_us"] = round(us, 2)
    pk = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))
    res["fused_floor_us_at_measured_peak"] = round(4 * n * n / pk["hbm_gbs"] / 1e3, 2)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
