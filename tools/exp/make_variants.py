"""Build kbench variants of the scan kernels for A/B timing on the GPU box.
Each variant is a copy of csrc/ with textual edits (timing experiments only:
some variants are deliberately inexact).  Output: scratch/kb_<name>."""
import os, shutil, subprocess, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
CS = "paper_conf_sigmod_heimelkm15_b200/csrc"
VARIANTS = {}
def variant(name):
    def deco(f):
        VARIANTS[name] = f
        return f
    return deco
def edit(path, old, new):
    s = open(path).read()
    assert old in s, (path, old[:60])
    open(path, "w").write(s.replace(old, new))

@variant("base")
def _base(d): pass

exec(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "variants.py")).read())

def build(name):
    d = os.path.join(ROOT, "scratch", "v_" + name)
    shutil.rmtree(d, ignore_errors=True)
    shutil.copytree(os.path.join(ROOT, CS), os.path.join(d, CS))
    os.makedirs(os.path.join(d, "tools"))
    shutil.copy(os.path.join(ROOT, "tools", "kbench.cu"), os.path.join(d, "tools"))
    VARIANTS[name](os.path.join(d, CS))
    out = os.path.join(ROOT, "scratch", "kb_" + name)
    r = subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
                        "-diag-suppress", "1886", "-o", out, os.path.join(d, "tools", "kbench.cu")],
                       capture_output=True, text=True)
    return name, r.returncode, r.stderr[-2000:]

names = sys.argv[1:] or list(VARIANTS)
with ThreadPoolExecutor(8) as ex:
    for name, rc, err in ex.map(build, names):
        print(name, "ok" if rc == 0 else "FAILED\n" + err)
