"""Build libddq.so in-tree with nvcc for sm_100a (no torch types in the ABI)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
SO = os.path.join(HERE, "libddq.so")
SOURCES = ["transfer.cu", "filter.cu", "dense.cu", "agg.cu", "scan.cu", "star.cu", "kernels.cu", "ops.cu", "engine.cpp",
           "driver.cpp", "dist.cpp", "cluster.cpp"]
HEADERS = ["device_common.cuh", "ops_internal.h", "engine.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [
        os.path.join(HERE, "..", "include", "ddq.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return SO
    objs = []
    builddir = os.path.join(HERE, "build")
    os.makedirs(builddir, exist_ok=True)
    hdr_t = max(os.path.getmtime(d) for d in [os.path.join(CSRC, f) for f in HEADERS] + [
        os.path.join(HERE, "..", "include", "ddq.h")])
    for src in SOURCES:
        obj = os.path.join(builddir, src + ".o")
        objs.append(obj)
        if not force and os.path.exists(obj) and os.path.getmtime(obj) > max(
                hdr_t, os.path.getmtime(os.path.join(CSRC, src))):
            continue  # object up to date
        cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3",
               "-Xptxas", "-v" if verbose else "-O3", "-x", "cu", "-c", os.path.join(CSRC, src), "-o", obj]
        if not src.endswith(".cu"):
            cmd = ["g++", "-O3", "-std=c++17", "-fPIC", "-Wall", "-I/usr/local/cuda/include", "-c",
                   os.path.join(CSRC, src), "-o", obj]
        subprocess.check_call(cmd)
    tmp = SO + ".tmp"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lpthread", "-ldl", "-Xlinker", "--no-undefined"])
    os.replace(tmp, SO)
    return SO


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(SO)
