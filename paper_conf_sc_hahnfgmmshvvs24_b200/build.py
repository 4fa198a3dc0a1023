"""Build libmdnorm.so (the C-ABI library of include/mdnorm.h) in-tree with nvcc for sm_100a."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libmdnorm.so")
INCLUDE = os.path.join(ROOT, "include")

NVCC_FLAGS = [
    "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
    # geometry must be bit-identical to the fp64 definition: no mul+add contraction anywhere
    # (the code also uses explicit __dmul_rn/__dadd_rn intrinsics; this is the guard)
    "--fmad=false",
    # host side: the flux cell table evaluates the device's U(x) expression (mdn_api.cu)
    "-Xcompiler", "-ffp-contract=off",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall", "-shared", "-cudart", "static",
]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    deps = sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(INCLUDE, "mdnorm.h"), __file__]
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, out: str | None = None,
          defines: tuple = ()) -> str:
    """Compile libmdnorm.so: every .cu to an object in parallel (relocatable device code is not
    needed: each translation unit owns its kernels), then one shared-library link.  out/defines
    build an experimental variant elsewhere (tools/)."""
    target = out or LIB
    if out is None and not force and not _stale():
        return LIB
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    tag = f".tmp{os.getpid()}_{os.path.basename(target)}"
    objs, procs = [], []
    for src in sources():
        obj = os.path.join(os.path.dirname(target), os.path.basename(src) + tag + ".o")
        cmd = [nvcc, *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-I", INCLUDE, "-c", "-o", obj, src]
        cmd.remove("-shared")
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
            print(" ".join(cmd), file=sys.stderr)
        objs.append(obj)
        procs.append(subprocess.Popen(cmd))
    try:
        bad = [p.args for p in procs if p.wait() != 0]
        if bad:
            raise subprocess.CalledProcessError(1, bad[0])
        tmp = target + tag
        link = [nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-cudart", "static",
                "-Xcompiler", "-fPIC", "-o", tmp, *objs]
        subprocess.check_call(link)
        os.replace(tmp, target)
    finally:
        for o in objs:
            if os.path.exists(o):
                os.remove(o)
    return target


if __name__ == "__main__":
    build(force=True, verbose="-v" in sys.argv)
    print(LIB)
