#!/usr/bin/env python
"""Summarise ncu reports into profiles/ (JSON + a short markdown table).

    python tools/ncu_summary.py --out profiles/ncu_summary.json \
        --full gpurun_out/prof_tma_r1c.ncu-rep [--full ...] \
        --launches gpurun_out/launches_r1a.csv

--full: `ncu --set full` captures (per-launch metrics of the profiled kernels);
--launches: the `--metrics gpu__time_duration.sum` launch list of a bench run.
The first --full report's first kernel is recorded as the dominant kernel (its DRAM
bytes per launch feed bench.py's roofline "traffic").
"""
from __future__ import annotations

import argparse
import csv
import io
import json
import subprocess
from collections import defaultdict

METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
    "launch__shared_mem_per_block_dynamic", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "lts__t_bytes.sum", "smsp__sass_inst_executed_op_branch.sum", "smsp__thread_inst_executed_pred_on.sum",
    "smsp__thread_inst_executed.sum", "smsp__inst_executed_pipe_alu.sum", "smsp__inst_executed_pipe_fma.sum",
    "smsp__inst_executed_pipe_lsu.sum", "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
    "smsp__pcsamp_warps_issue_stalled_barrier", "smsp__pcsamp_warps_issue_stalled_wait",
]

UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1.0,
              "msecond": 1e3, "ns": 1e-3, "us": 1.0, "ms": 1e3}


def raw_rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m in METRICS:
            if m in hdr:
                i = hdr.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                u = units[i]
                if u in ("byte", "Kbyte", "Mbyte", "Gbyte"):
                    v *= UNIT_SCALE[u]
                    m = m + " [bytes]"
                elif u in ("nsecond", "usecond", "msecond", "ns", "us", "ms"):
                    v *= UNIT_SCALE[u]
                    m = m + " [us]"
                d[m] = v
        res.append(d)
    return res


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    per = defaultdict(list)
    for r in rows:
        if "Kernel Name" in r and "Metric Value" in r:
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr):
            continue
        if r[hdr.index("Metric Name")] != "gpu__time_duration.sum":
            continue
        unit = r[hdr.index("Metric Unit")]
        v = float(r[hdr.index("Metric Value")].replace(",", "")) * UNIT_SCALE.get(unit, 1.0)
        per[r[hdr.index("Kernel Name")]].append(v)
    tot = sum(sum(v) for v in per.values())
    return {k: {"launches": len(v), "mean_us": sum(v) / len(v), "share": sum(v) / tot} for k, v in per.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", required=True)
    ap.add_argument("--full", action="append", default=[])
    ap.add_argument("--launches", default=None)
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    res = {"note": a.note, "reports": {}}
    for rep in a.full:
        res["reports"][rep] = raw_rows(rep)
    if a.full:
        k0 = res["reports"][a.full[0]][0]
        rb = k0.get("dram__bytes_read.sum [bytes]", 0)
        wb = k0.get("dram__bytes_write.sum [bytes]", 0)
        res["dominant_kernel"] = {"kernel": k0["kernel"], "dram_bytes_per_launch": rb + wb,
                                  "dram_read": rb, "dram_write": wb,
                                  "ncu_duration_us": k0.get("gpu__time_duration.sum [us]")}
    if a.launches:
        res["launch_list"] = launches(a.launches)
    json.dump(res, open(a.out, "w"), indent=1)
    md = a.out.rsplit(".", 1)[0] + ".md"
    with open(md, "w") as f:
        f.write(f"# ncu summary ({a.note})\n\n")
        for rep, ks in res["reports"].items():
            f.write(f"## {rep}\n\n| kernel | us | DRAM rd MB | DRAM wr MB | DRAM % | regs | warps act % | issue % |\n"
                    "|---|---|---|---|---|---|---|---|\n")
            for k in ks:
                f.write(f"| {k['kernel'][:70]} | {k.get('gpu__time_duration.sum [us]', 0):.2f} | "
                        f"{k.get('dram__bytes_read.sum [bytes]', 0) / 1e6:.1f} | "
                        f"{k.get('dram__bytes_write.sum [bytes]', 0) / 1e6:.1f} | "
                        f"{k.get('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 0):.1f} | "
                        f"{k.get('launch__registers_per_thread', 0):.0f} | "
                        f"{k.get('sm__warps_active.avg.pct_of_peak_sustained_active', 0):.1f} | "
                        f"{k.get('smsp__issue_active.avg.pct_of_peak_sustained_active', 0):.1f} |\n")
            f.write("\n")
        if "launch_list" in res:
            f.write("## launch list (cold-cache, serialised: compare shares)\n\n| kernel | launches | mean us | share |\n"
                    "|---|---|---|---|\n")
            for k, v in sorted(res["launch_list"].items(), key=lambda kv: -kv[1]["share"]):
                f.write(f"| {k[:80]} | {v['launches']} | {v['mean_us']:.2f} | {v['share']:.3f} |\n")
    print(json.dumps(res.get("dominant_kernel", {}), indent=1))


if __name__ == "__main__":
    main()
