#!/usr/bin/env python
"""Timing of the cfg3 u8 operators (Sobel dx/dy/mag, Laplace 5x5, Harris) on 4096^2,
Mirror, one JSON line per (variant, setting): CUDA graph of 12 launches over 6 rotating
buffer sets, CUDA events.  Settings: --override WX,TY (streaming launch shape), --env.

    python tools/bench_u8.py --variant warp --variant naive --override 4,8
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ipps_qiaoth21_b200 as isp  # noqa: E402
import synth  # noqa: E402
import numpy as np  # noqa: E402

G5 = np.outer(synth.binomial_row(5), synth.binomial_row(5)).astype(np.int32)


def timed(fn, R=12, reps=20):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for i in range(3):
            fn(i)
    torch.cuda.synchronize()
    plan = isp.isp_last_plan()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(R):
            fn(i)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        g.replay()
        e0.record(s)
        for _ in range(reps):
            g.replay()
        e1.record(s)
    torch.cuda.synchronize()
    return 1e3 * e0.elapsed_time(e1) / (R * reps), plan


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--variant", action="append", default=[])
    ap.add_argument("--override", action="append", default=[""])
    ap.add_argument("--size", type=int, default=4096)
    ap.add_argument("--mode", default="mirror")
    ap.add_argument("--env", action="append", default=[], help="KEY=VAL[,KEY=VAL] settings, one line each")
    ap.add_argument("--only", default="", help="comma list of sobel,laplace,harris")
    a = ap.parse_args()
    n, nb = a.size, 6
    imgs = [torch.from_numpy(synth.uniform_u8(n, n, 3 + i)).cuda() for i in range(nb)]
    dxs = [torch.empty((n, n), dtype=torch.int16, device="cuda") for _ in range(nb)]
    dys = [torch.empty_like(d) for d in dxs]
    o1 = [torch.empty_like(i) for i in imgs]
    o2 = [torch.empty_like(i) for i in imgs]
    o3 = [torch.empty_like(i) for i in imgs]
    for i in range(nb):
        isp.isp_sobel_u8(imgs[i], a.mode, dx=dxs[i], dy=dys[i], mag=o1[i])
    settings = [("", ov) for ov in a.override] + [(e, "") for e in a.env]
    for env, ov in settings:
        keys = []
        for kv in filter(None, env.split(",")):
            k, val = kv.split("=")
            os.environ[k] = val
            keys.append(k)
        if ov:
            isp.isp_set_launch_override(*map(int, ov.split(",")))
        for v in a.variant or ["auto"]:
            r = {}
            for name, bpp, fn in [
                ("sobel", 6, lambda i: isp.isp_sobel_u8(imgs[i % nb], a.mode, dx=dxs[i % nb], dy=dys[i % nb],
                                                        mag=o1[i % nb], variant=v)),
                ("copy", 2, lambda i: o2[i % nb].copy_(imgs[i % nb])),   # torch copy of the same bytes
                ("gauss5", 2, lambda i: isp.isp_filter_u8(imgs[i % nb], G5, 256, a.mode, out=o2[i % nb], variant=v)),
                ("laplace", 2, lambda i: isp.isp_laplace5_u8(imgs[i % nb], a.mode, out=o2[i % nb], variant=v)),
                ("harris", 5, lambda i: isp.isp_harris_u8(dxs[i % nb], dys[i % nb], a.mode, out=o3[i % nb], variant=v)),
            ]:
                if a.only and name not in a.only.split(","):
                    continue
                us, plan = timed(fn)
                r[name] = {"us": round(us, 2), "gbs": round(bpp * n * n / us / 1e3, 1),
                           "plan": [plan["tile_w"], plan["tile_h"], plan["nx"], plan["ny"], plan["choice"]]}
            print(json.dumps({"variant": v, "override": ov, "env": env, "px_u8": os.environ.get("ISP_LIB_PATH", ""), **r}), flush=True)
        if ov:
            isp.isp_set_launch_override(0, 0)
        for k in keys:
            del os.environ[k]


if __name__ == "__main__":
    main()
