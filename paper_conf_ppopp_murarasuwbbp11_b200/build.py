"""Build libsg.so in-tree with nvcc for sm_100a (B200).

    python paper_conf_ppopp_murarasuwbbp11_b200/build.py [--force] [-v]

All kernels and the C ABI (include/sg.h) are compiled by nvcc
(-gencode arch=compute_100a,code=sm_100a -lineinfo -O3) into one shared
library next to this file; nothing is JIT-compiled at import time.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libsg.so")
# experiment build (build.py --exp): the product sources plus csrc/exp/*.cu with -DSG_EXP, into a separate
# library that only scripts/gpu_exp.sh loads (SG_LIB); the product libsg.so never contains csrc/exp
LIB_EXP = os.path.join(PKG, "libsg_exp.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", "--expt-relaxed-constexpr",
         "-Xptxas", "-v", "-Wno-deprecated-gpu-targets"]


def sources(exp: bool = False):
    return sorted(glob.glob(os.path.join(CSRC, "*.cu"))) + (sorted(glob.glob(os.path.join(CSRC, "exp", "*.cu")))
                                                             if exp else [])


def _stale(exp: bool = False) -> bool:
    lib = LIB_EXP if exp else LIB
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = sources(exp) + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "sg.h"), __file__]
    return any(os.path.getmtime(p) > t for p in deps)


def _deps(path, seen=None):
    """The file and every local header it includes (transitively)."""
    seen = set() if seen is None else seen
    if path in seen or not os.path.exists(path):
        return seen
    seen.add(path)
    with open(path) as f:
        for line in f:
            line = line.strip()
            if line.startswith("#include \""):
                name = line.split('"')[1]
                for d in (os.path.dirname(path), os.path.join(ROOT, "include")):
                    _deps(os.path.join(d, name), seen)
    return seen


def build(force: bool = False, verbose: bool = False, exp: bool = False) -> str:
    lib = LIB_EXP if exp else LIB
    if not force and not _stale(exp):
        return lib
    objdir = os.path.join(PKG, "build_exp" if exp else "build")
    os.makedirs(objdir, exist_ok=True)
    flag_str = " ".join(ARCH + ["-O3", "-lineinfo"])
    objs, procs = [], []
    for src in sources(exp):
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        objs.append(obj)
        if not force and os.path.exists(obj) and all(
                os.path.getmtime(p) <= os.path.getmtime(obj) for p in _deps(src) | {__file__}):
            continue  # object newer than the source and every header it includes
        cmd = [NVCC, *ARCH, *FLAGS, f'-DSG_BUILD_FLAGS="{flag_str}"', "-I", os.path.join(ROOT, "include"),
               *(["-DSG_EXP=1"] if exp else []), "-c", src, "-o", obj]
        procs.append((src, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)))
    logs = []
    failed = None
    for src, p in procs:
        out, _ = p.communicate()
        logs.append(f"== {os.path.basename(src)}\n{out}")
        with open(os.path.join(objdir, os.path.basename(src) + ".log"), "w") as f:
            f.write(out)
        if p.returncode != 0:
            sys.stderr.write(out)
            failed = src
    if failed:
        raise RuntimeError(f"nvcc failed on {failed}")
    with open(os.path.join(objdir, "ptxas.log"), "w") as f:  # every object's ptxas -v output
        for src in sources(exp):
            lp = os.path.join(objdir, os.path.basename(src) + ".log")
            if os.path.exists(lp):
                f.write(f"== {os.path.basename(src)}\n" + open(lp).read())
    tmp = lib + ".tmp"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart"])
    os.replace(tmp, lib)
    if verbose:
        print("\n".join(logs))
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, exp="--exp" in sys.argv))
