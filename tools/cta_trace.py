#!/usr/bin/env python
"""Per-CTA timeline of one TMA-staged launch (diagnostics, ISP_CTA_TRACE): which regions /
SMs finish last.  Prints one JSON summary per border mode.

    ISP_CTA_TRACE=1 python tools/cta_trace.py --mode clamp --mode constant
"""
import argparse
import ctypes
import json
import os
import sys
from collections import defaultdict

os.environ.setdefault("ISP_CTA_TRACE", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_qiaoth21_b200 as isp  # noqa: E402
import synth  # noqa: E402

RG = ["TL", "TR", "T", "BL", "BR", "B", "R", "L", "Body"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mode", action="append", default=[])
    ap.add_argument("--size", type=int, default=4096)
    ap.add_argument("--window", type=int, default=5)
    a = ap.parse_args()
    n = a.size
    b = synth.binomial_row(a.window).astype(np.float64)
    mask = (np.outer(b, b) / b.sum() ** 2).astype(np.float32)
    pairs = [(torch.from_numpy(synth.uniform_f32(n, n, 2)).cuda(), torch.empty((n, n), device="cuda")) for _ in range(6)]
    L = isp.lib()
    L.isp_debug_cta_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
    for mode in a.mode or ["clamp"]:
        for i in range(8):
            inp, out = pairs[i % 6]
            isp.isp_filter_ex(inp, mask, mode, 0.5, out=out, variant="tma")
        torch.cuda.synchronize()
        plan = isp.isp_last_plan()
        nct = plan["nx"] * plan["ny"]
        buf = np.zeros((nct, 4), dtype=np.uint64)
        assert L.isp_debug_cta_trace(buf.ctypes.data, nct) == 0
        sm = (buf[:, 0] & 0xFFFF).astype(int)
        rg = ((buf[:, 0] >> 16) & 0xFFFF).astype(int)
        t0 = buf[:, 3].astype(np.int64)  # after griddepcontrol.wait (work start)
        t1 = buf[:, 2].astype(np.int64)
        base = t0.min()
        s, e = (t0 - base) / 1e3, (t1 - base) / 1e3
        dur = e - s
        per_rg = {}
        for r in sorted(set(rg)):
            m = rg == r
            per_rg[RG[r]] = {"n": int(m.sum()), "dur_us_mean": round(float(dur[m].mean()), 2),
                             "dur_us_max": round(float(dur[m].max()), 2), "end_us_max": round(float(e[m].max()), 2)}
        sm_end = defaultdict(float)
        for k in range(nct):
            sm_end[sm[k]] = max(sm_end[sm[k]], e[k])
        ends = np.array(sorted(sm_end.values()))
        late = np.argsort(-e)[:10]
        print(json.dumps({"mode": mode, "ctas": int(nct), "span_us": round(float(e.max()), 2),
                          "start_us_max": round(float(s.max()), 2),
                          "dur_us": {"mean": round(float(dur.mean()), 2), "p10": round(float(np.percentile(dur, 10)), 2),
                                     "p90": round(float(np.percentile(dur, 90)), 2), "max": round(float(dur.max()), 2)},
                          "sm_end_us": {"min": round(float(ends.min()), 2), "median": round(float(np.median(ends)), 2),
                                        "max": round(float(ends.max()), 2)},
                          "regions": per_rg,
                          "latest": [{"rg": RG[rg[k]], "sm": int(sm[k]), "by": int((buf[k, 0] >> 32) & 0xFFFF),
                                      "bx": int(buf[k, 0] >> 48), "start": round(float(s[k]), 2),
                                      "end": round(float(e[k]), 2)} for k in late]}), flush=True)


if __name__ == "__main__":
    main()
