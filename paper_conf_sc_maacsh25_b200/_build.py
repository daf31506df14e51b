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
    import time
    t_start = time.time()
    bdir = os.path.join(HERE, "build" if not defines else "build_" + "_".join(d.strip("-D").replace("=", "") for d in defines))
    os.makedirs(bdir, exist_ok=True)
    jobs = []
    for cu in sorted(glob.glob(os.path.join(CSRC, "*.cu"))):
        o = os.path.join(bdir, os.path.basename(cu) + ".o")
        cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-fopenmp", "-Xptxas", "-v",
               "-I", os.path.join(ROOT, "include"), *defines, "-c", cu, "-o", o]
        jobs.append((cu, o, cmd))
    for cpp in sorted(glob.glob(os.path.join(CSRC, "*.cpp"))):
        o = os.path.join(bdir, os.path.basename(cpp) + ".o")
        cmd = ["g++", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-std=c++17",
               "-I", os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include", *defines, "-c", cpp, "-o", o]
        jobs.append((cpp, o, cmd))
    # translation units compile in parallel (wchain.cu alone takes minutes); an object newer
    # than its source and every header is reused
    hdrs = [h for h in _sources() if h.endswith((".h", ".cuh"))]
    hdr_t = max(os.path.getmtime(h) for h in hdrs)

    def fresh(src, o):
        return not force and os.path.exists(o) and os.path.getmtime(o) >= max(os.path.getmtime(src), hdr_t)

    procs = [(src, o, None if fresh(src, o) else
              subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True))
             for src, o, cmd in jobs]
    objs, logs = [], []
    for src, o, pr in procs:
        objs.append(o)
        if pr is None:
            continue
        out, err = pr.communicate()
        if pr.returncode != 0:
            raise RuntimeError(f"compile of {os.path.basename(src)} failed:\n{err}")
        if verbose:
            print(err)
        logs.append(f"==== {os.path.basename(src)}\n{err}")
    if logs:
        with open(os.path.join(bdir, "ptxas.log"), "a") as f:
            f.write("\n".join(logs))
    tmp = lib + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-Xcompiler", "-fopenmp", "-lgomp"]
    subprocess.check_call(cmd)
    os.replace(tmp, lib)
    # stamp the library with the build's start time: a source edited while it compiled
    # makes the next build() recompile
    os.utime(lib, (t_start, t_start))
    return lib


if __name__ == "__main__":
    build(force=True, verbose=True)
    print(LIB)
