#!/usr/bin/env python
"""Quick read of one ncu report (run here, no GPU): headline metrics, stall reasons and the
SASS opcode mix weighted by execution count.

    python tools/ncu_quick.py gpurun_out/prof.ncu-rep [--hot N]
"""
import collections
import csv
import io
import subprocess
import sys


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[2]


def main():
    rep = sys.argv[1]
    hot = int(sys.argv[3]) if len(sys.argv) > 3 and sys.argv[2] == "--hot" else 0
    h, v = raw(rep)
    get = lambda k: v[h.index(k)] if k in h else "-"
    for k in ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
              "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
              "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem"]:
        print(f"{k:60s} {get(k)}")
    st = [(k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""), float(v[i]))
          for i, k in enumerate(h) if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("ratio")]
    print("stalls:", ", ".join(f"{a} {b:.2f}" for a, b in sorted(st, key=lambda t: -t[1])[:8]))
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hh, data = rows[1], rows[2:]
    ia, isrc = hh.index("Instructions Executed"), hh.index("Source")
    tot, ops = 0, collections.Counter()
    for r in data:
        n = int(r[ia] or 0)
        tot += n
        t = r[isrc].split()
        if not t:
            continue
        op = t[1] if t[0].startswith("@") and len(t) > 1 else t[0]
        ops[op.split(".")[0]] += n
    print("inst", tot, " ".join(f"{k}:{100 * c / tot:.1f}%" for k, c in ops.most_common(16)))
    if hot:
        for r in data:
            if int(r[ia] or 0) >= hot:
                print(r[ia], r[isrc].strip()[:100])


if __name__ == "__main__":
    main()
