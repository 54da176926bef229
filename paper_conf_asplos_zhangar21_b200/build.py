"""Build libvf.so in-tree with nvcc for sm_100a (B200).

Each csrc/*.cu is one module (an app's classes, vTables and kernels must share
a module: P:607-615), compiled in parallel to build/*.o and linked with the
static CUDA runtime so the library loads without libcuda on CPU-only hosts
(driver entry points are fetched at run time via cudaGetDriverEntryPoint).
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build", "vf")
SO = os.path.join(PKG, "libvf.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-O2",
                "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include"), "-Xptxas", "-v"]


def _headers():
    return glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(ROOT, "include", "vf.h")]


# Float apps whose results must match the CPU oracle bit for bit: no FMA
# contraction (every FMA is an explicit fmaf in the source), IEEE div/sqrt.
PER_FILE = {"app_ray.cu": ["-fmad=false", "-prec-div=true", "-prec-sqrt=true", "-ftz=false"],
            "app_nbody.cu": ["-fmad=false", "-prec-div=true", "-prec-sqrt=true", "-ftz=false"],
            "app_stut.cu": ["-fmad=false", "-prec-div=true", "-prec-sqrt=true", "-ftz=false"],
            "app_collide.cu": ["-fmad=false", "-prec-div=true", "-prec-sqrt=true", "-ftz=false"]}


def _compile(src: str, obj: str, verbose: bool) -> str:
    cmd = ["nvcc"] + FLAGS + PER_FILE.get(os.path.basename(src), []) + ["-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
    return r.stderr if verbose else ""


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    hdr_time = max(os.path.getmtime(h) for h in _headers() + [__file__])
    jobs = []
    objs = []
    for s in srcs:
        o = os.path.join(BUILD, os.path.basename(s)[:-3] + ".o")
        objs.append(o)
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(os.path.getmtime(s), hdr_time):
            jobs.append((s, o))
    if jobs:
        with cf.ThreadPoolExecutor(max_workers=min(8, len(jobs))) as ex:
            for log in ex.map(lambda j: _compile(j[0], j[1], verbose), jobs):
                if log:
                    sys.stderr.write(log)
    if jobs or not os.path.exists(SO) or os.path.getmtime(SO) < max(os.path.getmtime(o) for o in objs):
        cmd = ["nvcc"] + ARCH + ["-shared", "-cudart", "static", "-o", SO] + objs
        subprocess.run(cmd, check=True)
    return SO


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(SO)
