#!/usr/bin/env python
"""DRAM traffic per launch of bench.py's dominant kernel, measured by ncu over a RANGE of
back-to-back launches (so the output write-backs of every launch are counted -- a single
isolated ncu kernel replay leaves up to L2-size of dirty output in L2 and under-counts
writes).  Writes profiles/<tag>_traffic_<workload>.json, which bench.py reports as
roofline.traffic together with the libisp.so digest it was measured on.

On the GPU box:
    python tools/ncu_traffic.py --tag r02 [--workload cfg2] [--launches 24]
(it re-runs itself under `ncu --replay-mode range`; the range is delimited with
cudaProfilerStart/Stop around the launches, after warm-up).
"""
import argparse
import csv
import hashlib
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def workload_run(a):
    import numpy as np
    import torch

    import paper_conf_ipps_qiaoth21_b200 as isp
    import synth
    if a.workload == "cfg2":
        n, win, modes = 4096, 5, ["clamp", "mirror", "repeat", "constant"]
    else:
        n, win, modes = 16384, 7, ["clamp", "repeat"]
    b = synth.binomial_row(win).astype(np.float64)
    mask = (np.outer(b, b) / b.sum() ** 2).astype(np.float32)
    npairs = 6 if n == 4096 else 2
    src = torch.from_numpy(synth.uniform_f32(n, n, 2)) if n == 4096 else torch.rand((n, n))
    pairs = [(src.cuda(), torch.empty((n, n), device="cuda")) for _ in range(npairs)]
    stream = torch.cuda.Stream()

    def launch(i):
        inp, out = pairs[i % npairs]
        isp.isp_filter_ex(inp, mask, modes[i % len(modes)], 0.5, out=out, variant=a.variant, stream=stream)

    with torch.cuda.stream(stream):
        for i in range(8):
            launch(i)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    with torch.cuda.stream(stream):
        for i in range(a.launches):
            launch(i)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(json.dumps({"plan": isp.isp_last_plan()}))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="r02")
    ap.add_argument("--workload", default="cfg2", choices=["cfg2", "cfg5"])
    ap.add_argument("--variant", default="auto")
    ap.add_argument("--launches", type=int, default=24)
    ap.add_argument("--inner", action="store_true")
    ap.add_argument("--out-dir", default=os.path.join(ROOT, "profiles"),
                    help="on the GPU box use gpurun_out/ (merged back), then copy into profiles/")
    a = ap.parse_args()
    if a.inner:
        workload_run(a)
        return
    metrics = "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"
    cmd = ["ncu", "--replay-mode", "range", "--clock-control", "none", "--metrics", metrics, "--csv",
           sys.executable, os.path.abspath(__file__), "--inner", "--workload", a.workload, "--variant", a.variant,
           "--launches", str(a.launches)]
    r = subprocess.run(cmd, capture_output=True, text=True)
    lines = [l for l in r.stdout.splitlines() if l.startswith('"')]
    vals = {}
    for row in csv.DictReader(io.StringIO("\n".join(lines))):
        name, unit, v = row.get("Metric Name"), row.get("Metric Unit"), row.get("Metric Value")
        if not name:
            continue
        v = float(v.replace(",", ""))
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
                 "msecond": 1e-3, "second": 1}.get(unit, 1)
        vals[name] = vals.get(name, 0.0) + v * scale
    if "dram__bytes_read.sum" not in vals:
        print(r.stdout[-3000:], r.stderr[-3000:], file=sys.stderr)
        sys.exit(1)
    lib = os.path.join(ROOT, "paper_conf_ipps_qiaoth21_b200", "libisp.so")
    out = {"workload": a.workload, "variant": a.variant, "launches": a.launches,
           "dram_read_bytes": vals["dram__bytes_read.sum"], "dram_write_bytes": vals["dram__bytes_write.sum"],
           "range_time_s": vals.get("gpu__time_duration.sum"),
           "dram_bytes_per_launch": (vals["dram__bytes_read.sum"] + vals["dram__bytes_write.sum"]) / a.launches,
           "dram_read_per_launch": vals["dram__bytes_read.sum"] / a.launches,
           "dram_write_per_launch": vals["dram__bytes_write.sum"] / a.launches,
           "libisp_sha16": hashlib.sha256(open(lib, "rb").read()).hexdigest()[:16],
           "how": "ncu --replay-mode range over `launches` back-to-back launches (modes cycled), after warm-up; "
                  "per launch = range total / launches"}
    path = os.path.join(a.out_dir, f"{a.tag}_traffic_{a.workload}.json")
    json.dump(out, open(path, "w"), indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
