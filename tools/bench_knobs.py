#!/usr/bin/env python
"""Launch-shape / pipeline experiments for one kernel family on the cfg2 workload
(4096^2 f32, 5x5 binomial), timed like bench.py's variant table (CUDA graphs of 12
launches over rotating buffer pairs, CUDA events).  Prints one JSON line per setting.

    python tools/bench_knobs.py --variant tma --mode clamp \
        --env ISP_STAGES=3 --env ISP_STAGES=6 --env ISP_DEBUG_STAGED=1
Each --env is one setting (comma-separated KEY=VAL pairs); "" = defaults.
"""
import argparse
import json
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
    ap.add_argument("--env", action="append", default=[""])
    ap.add_argument("--override", action="append", default=[], help="WX,TY launch override settings")
    ap.add_argument("--cycle", action="store_true", help="cycle the four border modes inside the graph")
    a = ap.parse_args()
    n = a.size
    b = synth.binomial_row(a.window).astype(np.float64)
    mask = (np.outer(b, b) / b.sum() ** 2).astype(np.float32)
    host = torch.from_numpy(synth.uniform_f32(n, n, 2))
    pairs = [(host.cuda(), torch.empty((n, n), device="cuda")) for _ in range(6)]
    stream = torch.cuda.Stream()
    settings = [(e, None) for e in a.env] + [("", o) for o in a.override]
    for env, ov in settings:
        keys = []
        for kv in filter(None, env.split(",")):
            k, v = kv.split("=")
            os.environ[k] = v
            keys.append(k)
        if ov:
            wx, ty = map(int, ov.split(","))
            isp.isp_set_launch_override(wx, ty)
        R, reps = 12, 40

        modes = ["clamp", "mirror", "repeat", "constant"]

        def launch(i):
            inp, out = pairs[i % 6]
            m = modes[i % 4] if a.cycle else a.mode
            isp.isp_filter_ex(inp, mask, m, 0.5, out=out, variant=a.variant, stream=stream)

        with torch.cuda.stream(stream):
            for i in range(3):
                launch(i)
        torch.cuda.synchronize()
        plan = isp.isp_last_plan()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=stream):
            for i in range(R):
                launch(i)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            g.replay()
            e0.record(stream)
            for _ in range(reps):
                g.replay()
            e1.record(stream)
        torch.cuda.synchronize()
        us = 1e3 * e0.elapsed_time(e1) / (R * reps)
        print(json.dumps({"env": env, "override": ov, "variant": a.variant, "mode": "cycle" if a.cycle else a.mode,
                          "us": round(us, 3),
                          "gbs": round(8 * n * n / (us * 1e-6) / 1e9, 1),
                          "plan": {k: plan[k] for k in ("tile_w", "tile_h", "nx", "ny", "choice")}}), flush=True)
        for k in keys:
            del os.environ[k]
        if ov:
            isp.isp_set_launch_override(0, 0)


if __name__ == "__main__":
    main()
