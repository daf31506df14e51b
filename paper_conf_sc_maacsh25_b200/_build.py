"""In-tree build of libspcg.so (sm_100a CUDA kernels + host setup + C ABI).

nvcc cross-compiles for sm_100a without a GPU, so this runs on the CPU box too.
"""
from __future__ import annotations

import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libspcg.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")) +
                  glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "spcg.h")])


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in _sources())


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """defines/out: experiment variants (e.g. -DSPCG_VGROUP=1 -> libspcg_v1.so, loaded
    with SPCG_LIB=...); the default build is libspcg.so."""
    lib = out or LIB
    if not force and not defines and out is None and not stale():
        return LIB
    bdir = os.path.join(HERE, "build" if not defines else "build_" + "_".join(d.strip("-D").replace("=", "") for d in defines))
    os.makedirs(bdir, exist_ok=True)
    objs = []
    for cu in sorted(glob.glob(os.path.join(CSRC, "*.cu"))):
        o = os.path.join(bdir, os.path.basename(cu) + ".o")
        cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
               "-I", os.path.join(ROOT, "include"), *defines, "-c", cu, "-o", o]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed:\n{r.stderr}")
        if verbose:
            print(r.stderr)
        with open(os.path.join(bdir, "ptxas.log"), "w") as f:
            f.write(r.stderr)
        objs.append(o)
    for cpp in sorted(glob.glob(os.path.join(CSRC, "*.cpp"))):
        o = os.path.join(bdir, os.path.basename(cpp) + ".o")
        cmd = ["g++", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-std=c++17",
               "-I", os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include", *defines, "-c", cpp, "-o", o]
        subprocess.check_call(cmd)
        objs.append(o)
    tmp = lib + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-Xcompiler", "-fopenmp", "-lgomp"]
    subprocess.check_call(cmd)
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    build(force=True, verbose=True)
    print(LIB)
