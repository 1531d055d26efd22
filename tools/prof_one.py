#!/usr/bin/env python
"""A few plain launches of one filter call, for ncu captures (no graphs, no timing).

    ncu --set full -k regex:k_staged -s 2 -c 1 python tools/prof_one.py --variant tma --mode clamp
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_qiaoth21_b200 as isp  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--variant", default="tma")
    ap.add_argument("--mode", default="clamp")
    ap.add_argument("--size", type=int, default=4096)
    ap.add_argument("--window", type=int, default=5)
    ap.add_argument("--launches", type=int, default=4)
    ap.add_argument("--op", default="gauss", choices=["gauss", "gauss_u8", "sobel", "laplace", "harris", "bilateral", "fused3"])
    a = ap.parse_args()
    n = a.size
    if a.op != "gauss":
        u8 = torch.from_numpy(synth.uniform_u8(n, n, 3)).cuda()
        dx = torch.empty((n, n), dtype=torch.int16, device="cuda")
        dy = torch.empty_like(dx)
        o8 = torch.empty_like(u8)
        f = torch.from_numpy(synth.uniform_f32(n, n, 4)).cuda()
        fo = torch.empty_like(f)
        isp.isp_sobel_u8(u8, a.mode, dx=dx, dy=dy, mag=o8)
        for _ in range(a.launches):
            if a.op == "sobel":
                isp.isp_sobel_u8(u8, a.mode, dx=dx, dy=dy, mag=o8, variant=a.variant)
            elif a.op == "laplace":
                isp.isp_laplace5_u8(u8, a.mode, out=o8, variant=a.variant)
            elif a.op == "fused3":
                lap, har = torch.empty_like(u8), torch.empty_like(u8)
                isp.isp_pipeline_cfg3_u8(u8, a.mode, mag=o8, lap=lap, harris=har, variant=a.variant)
            elif a.op == "gauss_u8":
                b5 = np.array([1, 4, 6, 4, 1], dtype=np.int32)
                isp.isp_filter_u8(u8, np.outer(b5, b5).astype(np.int32), 256, a.mode, out=o8, variant=a.variant)
            elif a.op == "harris":
                isp.isp_harris_u8(dx, dy, a.mode, out=o8, variant=a.variant)
            else:
                isp.isp_bilateral_f32(f, a.window, (a.window - 1) / 4.0, 0.1, a.mode, 0.5, out=fo, variant=a.variant)
        torch.cuda.synchronize()
        return
    b = synth.binomial_row(a.window).astype(np.float64)
    mask = (np.outer(b, b) / b.sum() ** 2).astype(np.float32)
    inp = torch.from_numpy(synth.uniform_f32(n, n, 2)).cuda()
    out = torch.empty_like(inp)
    for _ in range(a.launches):
        isp.isp_filter_ex(inp, mask, a.mode, 0.5, out=out, variant=a.variant)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
