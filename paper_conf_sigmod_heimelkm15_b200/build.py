"""Builds libkde.so (the C-ABI library, include/kde.h) in-tree for sm_100a.

nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo, one object per
translation unit compiled in parallel, linked against the NCCL that ships
with torch (site-packages/nvidia/nccl) so one libnccl is loaded per process.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
OBJ = os.path.join(HERE, "build", "obj")
LIB = os.path.join(HERE, "libkde.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_dirs():
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    cands = []
    if spec and spec.submodule_search_locations:
        for loc in spec.submodule_search_locations:
            cands.append(os.path.join(loc, "nccl"))
    for c in cands:
        if os.path.exists(os.path.join(c, "include", "nccl.h")):
            return os.path.join(c, "include"), os.path.join(c, "lib")
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("command failed:\n" + " ".join(cmd) + "\n" + r.stdout + r.stderr)
    return r


def build(force: bool = False, verbose: bool = False, jobs: int = 0) -> str:
    inc, libdir = nccl_dirs()
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    hdrs = glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        glob.glob(os.path.join(ROOT, "include", "*.h"))
    newest_hdr = max(os.path.getmtime(h) for h in hdrs)
    os.makedirs(OBJ, exist_ok=True)
    flags = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-I", inc, "-I",
                    os.path.join(ROOT, "include"), "--expt-relaxed-constexpr"]

    def comp(src):
        obj = os.path.join(OBJ, os.path.basename(src) + ".o")
        if not force and os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(src), newest_hdr):
            return obj, False
        _run(["nvcc"] + flags + ["-c", src, "-o", obj])
        return obj, True

    with ThreadPoolExecutor(max_workers=jobs or os.cpu_count() or 4) as ex:
        res = list(ex.map(comp, srcs))
    objs = [o for o, _ in res]
    rebuilt = any(b for _, b in res)
    if rebuilt or force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        _run(["nvcc"] + ARCH + ["-shared", "-o", LIB] + objs +
             ["-L", libdir, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + libdir, "-lcudart"])
        if verbose:
            print("linked", LIB, file=sys.stderr)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
