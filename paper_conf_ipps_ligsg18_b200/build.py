"""Build libptas_b200.so in-tree (nvcc, sm_100a).  Used by __graft_entry__.build()."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libptas_b200.so")
# experiment builds (A/B of compile-time knobs): PTAS_VARIANT=<name> with
# PTAS_EXTRA_FLAGS="-DX=Y ..." writes variants/<name>/libptas_b200.so; load it
# with PTAS_LIB=<path> (paper_conf_ipps_ligsg18_b200/_native.py)
VARIANT = os.environ.get("PTAS_VARIANT")
if VARIANT:
    LIB = os.path.join(ROOT, "variants", VARIANT, "libptas_b200.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    return sorted(glob.glob(os.path.join(HERE, "csrc", "*.cu")) + glob.glob(os.path.join(HERE, "csrc", "*.cpp")))


def _headers():
    return glob.glob(os.path.join(HERE, "csrc", "*.h")) + glob.glob(os.path.join(HERE, "csrc", "*.cuh")) + \
        [os.path.join(ROOT, "include", "ptas.h")]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in sources() + _headers())


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile each source to build/*.o (in parallel, only when stale), then link."""
    if not force and not stale():
        return LIB
    from concurrent.futures import ThreadPoolExecutor
    objdir = os.path.join(os.path.dirname(LIB), "build") if VARIANT else os.path.join(HERE, "build")
    os.makedirs(objdir, exist_ok=True)
    hdr_t = max(os.path.getmtime(h) for h in _headers())
    # stale objects of removed sources must not be linked
    for o in glob.glob(os.path.join(objdir, "*.o")):
        if os.path.basename(o)[:-2] not in {os.path.basename(x) for x in sources()}:
            os.remove(o)
    flags = [*ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3", "-I" + os.path.join(ROOT, "include"),
             *os.environ.get("PTAS_EXTRA_FLAGS", "").split()]
    if verbose:
        flags.append("-Xptxas=-v")

    def compile_one(src):
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        if not force and os.path.exists(obj) and os.path.getmtime(obj) > max(os.path.getmtime(src), hdr_t):
            return obj
        tmp = obj + f".tmp{os.getpid()}"
        cmd = [NVCC, *flags, "-c", src, "-o", tmp]
        if verbose:
            print(" ".join(cmd))
        subprocess.check_call(cmd)
        os.replace(tmp, obj)
        return obj

    srcs = sorted(sources(), key=lambda x: -os.path.getsize(x))
    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(compile_one, srcs))
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-Xcompiler", "-fPIC", "-o", tmp, *objs, "-ldl"])
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
