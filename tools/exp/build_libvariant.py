"""Build a tuning copy of libkde.so with KDE_TUNE_* macro overrides (timing
experiments only; bench.py picks it up through KDE_LIB_PATH).
Usage: python tools/exp/build_libvariant.py NAME 'MACRO=VALUE' ... -> scratch/lib_NAME.so
Only the scan translation units (plus kernels.cu when KDE_VARIANT_KERNELS=1) see the
macros; the other objects are the in-tree build's (run the normal build first)."""
import glob, os, subprocess, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
from paper_conf_sigmod_heimelkm15_b200 import build as B  # noqa: E402

def main(name, macros):
    inc, libdir = B.nccl_dirs()
    out = os.path.join(ROOT, "scratch", "obj_" + name)
    os.makedirs(out, exist_ok=True)
    flags = B.ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-I", inc, "-I",
                      os.path.join(ROOT, "include"), "--expt-relaxed-constexpr", "-diag-suppress", "1886"]
    flags += ["-D" + m for m in macros]
    scan_srcs = sorted(glob.glob(os.path.join(B.CSRC, "scan_*.cu")))
    if os.environ.get("KDE_VARIANT_KERNELS") == "1":
        scan_srcs.append(os.path.join(B.CSRC, "kernels.cu"))
    def comp(src):
        obj = os.path.join(out, os.path.basename(src) + ".o")
        B._run(["nvcc"] + flags + ["-c", src, "-o", obj])
        return obj
    with ThreadPoolExecutor(os.cpu_count() or 4) as ex:
        objs = list(ex.map(comp, scan_srcs))
    mine = {os.path.basename(x) + ".o" for x in scan_srcs}
    base = [o for o in glob.glob(os.path.join(B.OBJ, "*.o")) if not os.path.basename(o).startswith("scan_")
            and os.path.basename(o) not in mine]
    lib = os.path.join(ROOT, "variants", f"lib_{name}.so")
    os.makedirs(os.path.dirname(lib), exist_ok=True)
    B._run(["nvcc"] + B.ARCH + ["-shared", "-o", lib] + objs + base +
           ["-L", libdir, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + libdir, "-lcudart"])
    print(lib)

if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2:])
