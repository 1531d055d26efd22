#!/usr/bin/env python
"""Build an experiment variant of libisp.so: csrc/ with some files replaced, only the
named units recompiled, linked with the in-tree objects.  Load it with ISP_LIB_PATH.

    python tools/exp_lib.py --name old --replace isp_staged.cuh=/tmp/old/isp_staged.cuh --units u_sep_f32_5
"""
import argparse
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_qiaoth21_b200 import build as B  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--name", required=True)
    ap.add_argument("--replace", action="append", default=[])
    ap.add_argument("--units", action="append", default=[])
    ap.add_argument("--define", action="append", default=[])
    ap.add_argument("--all", action="store_true", help="recompile every unit")
    a = ap.parse_args()
    if a.all:
        a.units = sorted(f[:-3] for f in os.listdir(B.CSRC) if f.endswith(".cu"))
    B.build()
    tmp = tempfile.mkdtemp()
    src = os.path.join(tmp, "a", "b", "csrc")  # api.cu includes ../../include/isp.h
    shutil.copytree(B.CSRC, src)
    shutil.copytree(B.INCLUDE, os.path.join(tmp, "a", "include"))
    for r in a.replace:
        k, v = r.split("=")
        shutil.copy(v, os.path.join(src, k))
    inc, lib = B.nccl_paths()
    objs = {os.path.basename(o)[:-2]: os.path.join(B.OBJ, o) for o in os.listdir(B.OBJ) if o.endswith(".o")}
    from concurrent.futures import ThreadPoolExecutor

    def one(u):
        o = os.path.join(tmp, u + ".o")
        subprocess.run([B.nvcc(), *B.ARCH, *B.NVCC_FLAGS, *[f"-D{d}" for d in a.define], "-I", inc, "-I", B.INCLUDE,
                        "-c", os.path.join(src, u + ".cu"), "-o", o], check=True, capture_output=True)
        return u, o

    with ThreadPoolExecutor(os.cpu_count()) as ex:
        for u, o in ex.map(one, a.units):
            objs[u] = o
    os.makedirs(os.path.join(ROOT, "exp_libs"), exist_ok=True)
    out = os.path.join(ROOT, "exp_libs", f"libisp_{a.name}.so")
    subprocess.run([B.nvcc(), *B.ARCH, "-shared", "-o", out, *objs.values(), "-L", lib, "-l:libnccl.so.2",
                    "-Xlinker", f"-rpath={lib}", "-cudart", "static"], check=True)
    print(out)


if __name__ == "__main__":
    main()
