#!/usr/bin/env python
"""Per-kernel measurements of every SURVEY.md 8(a) row on BASELINE.json's configs.

Same methodology as bench.py's variant table: a CUDA graph of R launches over rotating
input/output buffers (>= 2x L2 in total unless the config is tiny), replayed `reps` times,
CUDA events on the launch stream.  Prints one JSON document (saved under profiles/).

    python tools/bench_suite.py [--quick] > profiles/r01_suite.json
"""
from __future__ import annotations

import argparse
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_qiaoth21_b200 as isp  # noqa: E402
import synth  # noqa: E402

MODES = ["clamp", "mirror", "repeat", "constant"]
L2_BYTES = 126 * 2 ** 20


def peaks():
    try:
        return json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                           "MEASURED_PEAKS.json")))
    except Exception:
        return {}


HBM = peaks().get("hbm_gbs", 6650.0)


def nbuf_for(bytes_per_pair):
    return max(2, min(12, math.ceil(2 * L2_BYTES / max(bytes_per_pair, 1)) + 1))


def time_launch(fn, nbuf, R=12, reps=20):
    """fn(i) launches one kernel on buffer set i % nbuf on the current stream."""
    stream = torch.cuda.Stream()
    with torch.cuda.stream(stream):
        for i in range(max(2, min(nbuf, R))):   # every buffer once: per-buffer host state (texture objects) exists before capture
            fn(i)
    torch.cuda.synchronize()
    plan = isp.isp_last_plan()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=stream):
        for i in range(R):
            fn(i)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        g.replay()
        a.record(stream)
        for _ in range(reps):
            g.replay()
        b.record(stream)
    torch.cuda.synchronize()
    return 1e3 * a.elapsed_time(b) / (R * reps), plan


def binomial_f32(m):
    b = synth.binomial_row(m).astype(np.float64)
    return (np.outer(b, b) / b.sum() ** 2).astype(np.float32)


def rec(us, px, nbytes, plan=None, extra=None):
    d = {"us": round(us, 3), "mpix_s": round(px / us, 1), "gbs": round(nbytes / (us * 1e-6) / 1e9, 1),
         "hbm_frac": round(nbytes / (us * 1e-6) / 1e9 / HBM, 4)}
    if plan is not None:
        d["choice"] = {0: "auto", 1: "block", 2: "warp", 3: "naive", 4: "tma"}[plan["choice"]]
        d["G"] = plan["g"]
    if extra:
        d.update(extra)
    return d


def cfg1():
    n = 64
    img = torch.from_numpy(synth.uniform_u8(n, n, 1)).cuda()
    out = torch.empty_like(img)
    b = synth.binomial_row(3)
    mask, div = np.outer(b, b).astype(np.int32), int(b.sum()) ** 2
    res = {}
    for v in ["auto", "tma", "warp", "naive"]:
        us, plan = time_launch(lambda i: isp.isp_filter_u8(img, mask, div, "clamp", out=out, variant=v), 1)
        res[v] = rec(us, n * n, 2 * n * n, plan, {"degenerate": plan["degenerate"]})
    return {"config": "3x3 Gaussian u8 64x64 clamp (latency-bound: 8 KB)", "variants": res}


def cfg2():
    n = 4096
    nb = nbuf_for(8 * n * n)
    ins = [torch.from_numpy(synth.uniform_f32(n, n, 2)).cuda() for _ in range(1)] * nb
    outs = [torch.empty((n, n), device="cuda") for _ in range(nb)]
    ins = [ins[0].clone() for _ in range(nb)]
    res = {}
    for mwin in (5,):
        mask = binomial_f32(mwin)
        for m in MODES:
            res[m] = {}
            for v in ["tma", "warp", "block", "naive"]:
                us, plan = time_launch(lambda i: isp.isp_filter_ex(ins[i % nb], mask, m, 0.5, out=outs[i % nb],
                                                                   variant=v), nb)
                res[m][v] = rec(us, n * n, 8 * n * n, plan)
            res[m]["speedup_isp_vs_naive"] = res[m]["naive"]["us"] / res[m]["tma"]["us"]
    # non-separable 5x5 mask (2-D path) for reference
    rnd = np.random.default_rng(1).random((5, 5)).astype(np.float32)
    us, plan = time_launch(lambda i: isp.isp_filter_ex(ins[i % nb], rnd, "clamp", 0.5, out=outs[i % nb],
                                                       variant="auto"), nb)
    res["clamp_2d_mask"] = rec(us, n * n, 8 * n * n, plan)
    return {"config": "5x5 Gaussian f32 4096^2, 4 modes, ISP vs naive", "per_mode": res}


def cfg3():
    n = 4096
    nb = nbuf_for(15 * n * n)
    img = [torch.from_numpy(synth.structured_u8(n, n, 3)).cuda() for _ in range(1)][0]
    imgs = [img.clone() for _ in range(nb)]
    dxs = [torch.empty((n, n), dtype=torch.int16, device="cuda") for _ in range(nb)]
    dys = [torch.empty((n, n), dtype=torch.int16, device="cuda") for _ in range(nb)]
    mags = [torch.empty((n, n), dtype=torch.uint8, device="cuda") for _ in range(nb)]
    laps = [torch.empty((n, n), dtype=torch.uint8, device="cuda") for _ in range(nb)]
    hars = [torch.empty((n, n), dtype=torch.uint8, device="cuda") for _ in range(nb)]
    for i in range(nb):
        isp.isp_sobel_u8(imgs[i], "mirror", dx=dxs[i], dy=dys[i], mag=mags[i])
    res = {}
    for v in ["auto", "tma", "warp", "naive"]:
        r = {}
        us, plan = time_launch(lambda i: isp.isp_sobel_u8(imgs[i % nb], "mirror", dx=dxs[i % nb], dy=dys[i % nb],
                                                          mag=mags[i % nb], variant=v), nb)
        r["sobel_dx_dy_mag"] = rec(us, n * n, 6 * n * n, plan)
        us, plan = time_launch(lambda i: isp.isp_laplace5_u8(imgs[i % nb], "mirror", out=laps[i % nb], variant=v), nb)
        r["laplace5"] = rec(us, n * n, 2 * n * n, plan)
        us, plan = time_launch(lambda i: isp.isp_harris_u8(dxs[i % nb], dys[i % nb], "mirror", out=hars[i % nb],
                                                           variant=v), nb)
        r["harris"] = rec(us, n * n, 5 * n * n, plan)
        tot = sum(x["us"] for x in r.values())
        r["pipeline"] = rec(tot, n * n, 13 * n * n)
        res[v] = r
    # one-launch fusion (isp_pipeline_cfg3_u8): 1 B/px in, mag + lap + harris out
    fused = {}
    for v in ["auto", "naive"]:
        us, _ = time_launch(lambda i: isp.isp_pipeline_cfg3_u8(imgs[i % nb], "mirror", mag=mags[i % nb],
                                                               lap=laps[i % nb], harris=hars[i % nb], variant=v), nb)
        fused[v] = rec(us, n * n, 4 * n * n)
        us, _ = time_launch(lambda i: isp.isp_pipeline_cfg3_u8(imgs[i % nb], "mirror", mag=mags[i % nb],
                                                               lap=laps[i % nb], harris=hars[i % nb], dx=dxs[i % nb],
                                                               dy=dys[i % nb], variant=v), nb)
        fused[v + "_with_dx_dy"] = rec(us, n * n, 8 * n * n)
    fused["speedup_vs_3_launches"] = res["auto"]["pipeline"]["us"] / fused["auto"]["us"]
    return {"config": "Sobel + Laplace + Harris pipeline, 4096^2 u8, mirror (13 B/px: Sobel fused 6, Laplace 2, "
                      "Harris 5; fused: 4 B/px, 8 with dx/dy)", "variants": res, "fused": fused}


def cfg4(sweep=True):
    n = 2048
    nb = nbuf_for(8 * n * n)
    img = torch.from_numpy(synth.structured_f32(n, n, 4)).cuda()
    ins = [img.clone() for _ in range(nb)]
    outs = [torch.empty((n, n), device="cuda") for _ in range(nb)]
    clock_hz = 1.965e9
    mufu_peak = 16 * 148 * clock_hz          # ex2 per second

    def one(win, m, v):
        sd = max((win - 1) / 4.0, 0.5)
        us, plan = time_launch(lambda i: isp.isp_bilateral_f32(ins[i % nb], win, sd, 0.1, m, 0.5, out=outs[i % nb],
                                                               variant=v), nb, R=6, reps=5)
        nexp = win * win * n * n
        return rec(us, n * n, 8 * n * n, plan, {"ex2_per_s": nexp / (us * 1e-6),
                                                "mufu_frac": nexp / (us * 1e-6) / mufu_peak})

    res = {"win13": {m: {v: one(13, m, v) for v in ["auto", "tma", "warp", "naive"]} for m in MODES}}
    if sweep:
        sw = {}
        for m in MODES:
            rows = []
            for win in range(3, 32, 2):
                a = one(win, m, "auto")
                w = one(win, m, "warp")
                nv = one(win, m, "naive")
                t = one(win, m, "tma")
                rows.append({"win": win, "isp_us": w["us"], "naive_us": nv["us"], "speedup": nv["us"] / w["us"],
                             "tiled_us": t["us"], "tiled_mufu_frac": t["mufu_frac"], "auto_us": a["us"],
                             "G": a["G"], "auto_choice": a["choice"]})
            sp = np.array([r["speedup"] for r in rows])
            G = np.array([r["G"] for r in rows])
            pr = float(np.corrcoef(G, sp)[0, 1]) if np.std(G) > 0 and np.std(sp) > 0 else None
            sw[m] = {"rows": rows, "pearson_r_G_vs_speedup": pr}
        res["sweep"] = sw
    return {"config": "Bilateral f32 2048^2, 13x13, 4 modes; window sweep 3..31 (model G vs measured speedup)",
            "mufu_roofline": "16 ex2/clk/SM x 148 SMs x 1.965 GHz (SURVEY 8(d))", "results": res}


def cfg5():
    n = 16384
    img = torch.rand((n, n), device="cuda")
    outs = [torch.empty((n, n), device="cuda") for _ in range(2)]
    ins = [img, img.clone()]
    mask = binomial_f32(7)
    res = {}
    for m in ["clamp", "repeat"]:
        for v in ["auto", "naive"]:
            us, plan = time_launch(lambda i: isp.isp_filter_ex(ins[i % 2], mask, m, 0.0, out=outs[i % 2], variant=v),
                                   2, R=4, reps=10)
            res[f"{m}_{v}"] = rec(us, n * n, 8 * n * n, plan)
    return {"config": "16384^2 Gaussian 7x7 f32, single GPU (the strip path's per-rank kernel)", "results": res}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--only", default=None)
    a = ap.parse_args()
    out = {"hbm_peak_gbs": HBM, "device": torch.cuda.get_device_name(0)}
    for name, fn in [("cfg1", cfg1), ("cfg2", cfg2), ("cfg3", cfg3), ("cfg4", lambda: cfg4(not a.quick)),
                     ("cfg5", cfg5)]:
        if a.only and name not in a.only.split(","):
            continue
        out[name] = fn()
        print(f"[suite] {name} done", file=sys.stderr, flush=True)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
