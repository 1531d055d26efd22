#!/usr/bin/env python
"""Instruction, branch, predication and occupancy counters of ISP vs naive kernels
(the B200 analog of the paper's Table I (instruction counts)
and Table II (registers / occupancy)), and the model calibration of reading A19:

    n_kernel = I_isp / (m n px),   n_check = (I_naive - I_isp) / (4 m n px)

with I = smsp__thread_inst_executed.sum of one launch on an image of px pixels (the ISP
launch is dominated by its Body region; the naive launch checks every read).

On the GPU box:   python tools/ncu_counters.py --tag r02 --out-dir gpurun_out
It re-runs itself under ncu (one launch per case, every kernel profiled) and writes
<tag>_counters.json (+ .md table) with one record per case.
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "smsp__inst_executed.sum", "smsp__thread_inst_executed.sum", "smsp__thread_inst_executed_pred_on.sum",
    "smsp__sass_inst_executed_op_branch.sum", "smsp__sass_branch_targets_threads_divergent.sum",
    "smsp__inst_executed_pipe_alu.sum", "smsp__inst_executed_pipe_fma.sum", "smsp__inst_executed_pipe_xu.sum",
    "smsp__inst_executed_pipe_lsu.sum",
    "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
    "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__maximum_warps_per_active_cycle_pct",
]
MODES = ["clamp", "mirror", "repeat", "constant"]


def cases():
    """(label, family, m, n, px, make_and_launch) -- one launch each, in this order."""
    import numpy as np
    import torch

    import paper_conf_ipps_qiaoth21_b200 as isp
    import synth
    out = []
    n2 = 4096
    f = torch.from_numpy(synth.uniform_f32(n2, n2, 2)).cuda()
    fo = torch.empty_like(f)
    b5 = synth.binomial_row(5).astype(np.float64)
    g5 = (np.outer(b5, b5) / b5.sum() ** 2).astype(np.float32)
    r5 = np.random.default_rng(5).standard_normal((5, 5)).astype(np.float32)
    u8 = torch.from_numpy(synth.structured_u8(n2, n2, 3)).cuda()
    u8o = torch.empty_like(u8)
    dx = torch.empty((n2, n2), dtype=torch.int16, device="cuda")
    dy = torch.empty_like(dx)
    isp.isp_sobel_u8(u8, "mirror", dx=dx, dy=dy, mag=u8o)
    G5 = np.outer(synth.binomial_row(5), synth.binomial_row(5)).astype(np.int32)
    fb = torch.from_numpy(synth.structured_f32(2048, 2048, 4)).cuda()
    fbo = torch.empty_like(fb)
    px4, px2 = n2 * n2, 2048 * 2048
    for mode in MODES:
        for v in ["tma", "warp", "block", "naive"]:
            out.append((f"cfg2_gauss5_f32/{mode}/{v}", "sep_f32", 5, 5, px4,
                        lambda m=mode, v=v: isp.isp_filter_ex(f, g5, m, 0.5, out=fo, variant=v)))
        for v in ["warp", "naive"]:
            out.append((f"conv5_f32/{mode}/{v}", "conv_f32", 5, 5, px4,
                        lambda m=mode, v=v: isp.isp_filter_ex(f, r5, m, 0.5, out=fo, variant=v)))
            out.append((f"gauss5_u8/{mode}/{v}", "u8", 5, 5, px4,
                        lambda m=mode, v=v: isp.isp_filter_u8(u8, G5, int(G5.sum()), m, 7, out=u8o, variant=v)))
            out.append((f"sobel_u8/{mode}/{v}", "sobel", 3, 3, px4,
                        lambda m=mode, v=v: isp.isp_sobel_u8(u8, m, 7, dx=dx, dy=dy, mag=u8o, variant=v)))
            out.append((f"laplace5_u8/{mode}/{v}", "laplace", 5, 5, px4,
                        lambda m=mode, v=v: isp.isp_laplace5_u8(u8, m, 7, out=u8o, variant=v)))
            out.append((f"harris_i16/{mode}/{v}", "harris", 3, 3, px4,
                        lambda m=mode, v=v: isp.isp_harris_u8(dx, dy, m, 0, 0, out=u8o, variant=v)))
            out.append((f"atrous2_f32/{mode}/{v}", "atrous", 3, 3, px4,
                        lambda m=mode, v=v: isp.isp_atrous_f32(f, 2, m, 0.5, out=fo, variant=v)))
            out.append((f"bilateral13_f32/{mode}/{v}", "bilateral", 13, 13, px2,
                        lambda m=mode, v=v: isp.isp_bilateral_f32(fb, 13, 3.0, 0.1, m, 0.5, out=fbo, variant=v)))
        out.append((f"gauss5_u8/{mode}/tma", "u8", 5, 5, px4,
                    lambda m=mode: isp.isp_filter_u8(u8, G5, int(G5.sum()), m, 7, out=u8o, variant="tma")))
        out.append((f"bilateral13_f32/{mode}/tma", "bilateral", 13, 13, px2,
                    lambda m=mode: isp.isp_bilateral_f32(fb, 13, 3.0, 0.1, m, 0.5, out=fbo, variant="tma")))
    for v in ["tma", "warp", "naive"]:
        for op, fam, m in (("sobel_u8", "sobel", 3), ("laplace5_u8", "laplace", 5), ("harris_i16", "harris", 3)):
            def call(op=op, v=v):
                if op == "sobel_u8":
                    isp.isp_sobel_u8(u8, "mirror", 7, dx=dx, dy=dy, mag=u8o, variant=v)
                elif op == "laplace5_u8":
                    isp.isp_laplace5_u8(u8, "mirror", 7, out=u8o, variant=v)
                else:
                    isp.isp_harris_u8(dx, dy, "mirror", 0, 0, out=u8o, variant=v)
            out.append((f"cfg3_{op}/mirror/{v}", fam, m, m, px4, call))
    for v in ["auto", "naive"]:
        out.append((f"cfg3_fused/mirror/{v}", "fused", 5, 5, px4,
                    lambda v=v: isp.isp_pipeline_cfg3_u8(u8, "mirror", 7, 0, 0, variant=v)))
    return out


def inner(a):
    import torch
    cs = cases()
    torch.cuda.synchronize()
    torch.cuda.profiler.start()      # ncu --profile-from-start off: only the cases below
    labels = []
    for (label, fam, m, n, px, fn) in cs:
        fn()
        torch.cuda.synchronize()
        import paper_conf_ipps_qiaoth21_b200 as isp
        plan = isp.isp_last_plan()
        labels.append({"label": label, "family": fam, "m": m, "n": n, "px": px, "choice": plan["choice"],
                       "g": plan["g"], "degenerate": plan["degenerate"]})
    torch.cuda.profiler.stop()
    json.dump(labels, open(a.labels, "w"))


def markdown(out, tag):
    """Table I / Table II analog: per launch, per output pixel."""
    lines = [f"# ncu counters {tag}: ISP vs naive (Table I / II analog), one launch per row",
             "", "Per output pixel: thread instructions, branch instructions (thread-level), predicated-on share; "
             "registers, register occupancy limit (blocks / SM), achieved warps. `tools/ncu_counters.py`.", "",
             "| case | us | inst/px | branch/px | pred-on % | divergent branches | regs | occ. limit (regs) | warps active % |",
             "|---|---|---|---|---|---|---|---|---|"]
    for r in out["records"]:
        px = r["px"]
        ti = r["smsp__thread_inst_executed.sum"]
        lines.append("| {} | {:.1f} | {:.1f} | {:.2f} | {:.1f} | {:.0f} | {:.0f} | {:.0f} | {:.1f} |".format(
            r["label"], r["gpu__time_duration.sum"] / 1000.0, ti / px,
            r["smsp__sass_inst_executed_op_branch.sum"] * 32 / px,
            100.0 * r["smsp__thread_inst_executed_pred_on.sum"] / ti, r["smsp__sass_branch_targets_threads_divergent.sum"],
            r["launch__registers_per_thread"], r["launch__occupancy_limit_registers"],
            r["sm__warps_active.avg.pct_of_peak_sustained_active"]))
    lines += ["", "## Calibration (reading A19): n_kernel = I_isp / (m n px), n_check = (I_naive - I_isp) / (4 m n px)",
              "", "| family / mode | n_check | n_kernel | inst/px ISP | inst/px naive |", "|---|---|---|---|---|"]
    for k, v in sorted(out["calibration"].items()):
        lines.append(f"| {k} | {v['n_check']:.4f} | {v['n_kernel']:.4f} | {v['thread_inst_per_px_isp']:.1f} | "
                     f"{v['thread_inst_per_px_naive']:.1f} |")
    return "\n".join(lines) + "\n"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="r03")
    ap.add_argument("--out-dir", default=os.path.join(ROOT, "profiles"))
    ap.add_argument("--inner", action="store_true")
    ap.add_argument("--labels", default="/tmp/ncu_counter_labels.json")
    a = ap.parse_args()
    if a.inner:
        inner(a)
        return
    cmd = ["ncu", "--clock-control", "none", "--profile-from-start", "off", "--metrics", ",".join(METRICS),
           "--csv", "-k", "regex:^k_",
           sys.executable, os.path.abspath(__file__), "--inner", "--labels", a.labels]
    r = subprocess.run(cmd, capture_output=True, text=True)
    lines = [l for l in r.stdout.splitlines() if l.startswith('"')]
    per = {}
    order = []
    for row in csv.DictReader(io.StringIO("\n".join(lines))):
        kid = int(row["ID"])
        if kid not in per:
            per[kid] = {"kernel": row["Kernel Name"]}
            order.append(kid)
        v = row["Metric Value"].replace(",", "")
        try:
            v = float(v)
        except ValueError:
            pass
        per[kid][row["Metric Name"]] = v
        per[kid][row["Metric Name"] + "@unit"] = row["Metric Unit"]
    labels = json.load(open(a.labels))
    # every case is exactly one launch of one of the library's k_* kernels
    recs = [per[k] for k in order]
    if len(recs) != len(labels):
        print(f"warning: {len(recs)} profiled isp kernels vs {len(labels)} cases", file=sys.stderr)
    res = []
    for lab, rec in zip(labels, recs):
        rec.update(lab)
        res.append(rec)
    # calibration (reading A19): per (family, mode) from the warp (ISP) and naive launches
    calib = {}
    for rec in res:
        fam_mode = rec["label"].rsplit("/", 1)[0]
        calib.setdefault(fam_mode, {})[rec["label"].rsplit("/", 1)[1]] = rec
    cal = {}
    for key, d in calib.items():
        if "warp" in d and "naive" in d:
            r0 = d["warp"]
            mn, px = r0["m"] * r0["n"], r0["px"]
            ii, iN = d["warp"]["smsp__thread_inst_executed.sum"], d["naive"]["smsp__thread_inst_executed.sum"]
            cal[key] = {"family": r0["family"], "n_kernel": ii / (mn * px), "n_check": (iN - ii) / (4 * mn * px),
                        "thread_inst_per_px_isp": ii / px, "thread_inst_per_px_naive": iN / px}
    out = {"records": res, "calibration": cal, "metrics": METRICS}
    path = os.path.join(a.out_dir, f"{a.tag}_counters.json")
    json.dump(out, open(path, "w"), indent=1)
    open(path[:-5] + ".md", "w").write(markdown(out, a.tag))
    print(f"wrote {path}: {len(res)} records, {len(cal)} calibration rows")
    if r.returncode != 0:
        print(r.stderr[-3000:], file=sys.stderr)


if __name__ == "__main__":
    main()
