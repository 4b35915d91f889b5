"""Builds libpesto.so in-tree for sm_100a (nvcc for the kernels, g++ for the host runtime)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INC = os.path.join(ROOT, "include")
OUT = os.path.join(HERE, "libpesto.so")
BUILD = os.path.join(HERE, "build")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]

CU_SOURCES = ["kernels.cu", "eval32.cu", "nondelay.cu", "roofs.cu"]
CPP_SOURCES = ["graph.cpp", "layout.cpp", "search.cpp", "coarsen.cpp"]
HEADERS = ["internal.h", "host.h", "layout_format.h", "moves.cuh", "device_common.cuh",
           "feasibility.cuh", "uni_push_ptx.inc", "fast_walk_ptx.inc"]


def _stale() -> bool:
    if not os.path.exists(OUT):
        return True
    t = os.path.getmtime(OUT)
    srcs = [os.path.join(CSRC, f) for f in CU_SOURCES + CPP_SOURCES + HEADERS]
    srcs += [os.path.join(INC, "pesto.h"), os.path.abspath(__file__)]
    return any(os.path.getmtime(s) > t for s in srcs)


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
        raise RuntimeError(f"build failed: {cmd[0]} {cmd[-1]}")
    return r


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return OUT
    os.makedirs(BUILD, exist_ok=True)
    jobs = []
    for f in CU_SOURCES:
        o = os.path.join(BUILD, f + ".o")
        cmd = [NVCC, *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC",
               "-Xptxas", "-v" if verbose else "-O3", "-I", INC, "-I", CSRC, "-c",
               os.path.join(CSRC, f), "-o", o]
        jobs.append((cmd, o))
    for f in CPP_SOURCES:
        o = os.path.join(BUILD, f + ".o")
        jobs.append((["g++", "-O2", "-std=c++17", "-fPIC", "-Wall", "-I",
                      os.path.join(CUDA, "include"), "-I", INC, "-I", CSRC, "-c",
                      os.path.join(CSRC, f), "-o", o], o))
    # the translation units are independent: compile them concurrently
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=min(len(jobs), os.cpu_count() or 1)) as ex:
        results = list(ex.map(lambda jc: _run(jc[0]), jobs))
    if verbose:
        for r in results:
            sys.stderr.write(r.stderr)
    objs = [o for _, o in jobs]
    tmp = OUT + ".tmp"
    _run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-ldl", "-lpthread",
          "-lrt"])
    os.replace(tmp, OUT)
    return OUT


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
