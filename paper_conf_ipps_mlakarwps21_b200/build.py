"""Build librcm.so (sm_100a) in-tree with nvcc.  No torch at build time."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "librcm.so")
SOURCES = ["rcm.cu"]
HEADERS = ["rcm_device.cuh", "rcm_batch.cuh", "rcm_workers.cuh", "rcm_lookback.cuh", "rcm_components.cuh", "rcm_leveled.cuh"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC,-O2", "-cudart", "static", "-shared",
         "-Xptxas", "-warn-spills"]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(HERE, "..", "include", "rcm.h"))
    deps.append(os.path.abspath(__file__))
    return any(os.path.getmtime(d) > t for d in deps if os.path.exists(d))


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    extra = [f"-DRCM_THREADS={os.environ['RCM_THREADS']}"] if os.environ.get("RCM_THREADS") else []
    if os.environ.get("RCM_DISC_U"):
        extra.append(f"-DRCM_DISC_U={os.environ['RCM_DISC_U']}")
    if os.environ.get("RCM_TRACE"):
        extra.append("-DRCM_TRACE")
    cmd = [NVCC, *FLAGS, *extra, "-o", tmp, *[os.path.join(CSRC, s) for s in SOURCES]]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


CPU_LIB = os.path.join(HERE, "libcpubatch.so")
CPU_SRC = os.path.join(CSRC, "cpu_batch.cpp")
CXX = os.environ.get("CXX", "g++")


def build_cpu(force: bool = False) -> str:
    """Host CPU-BATCH (NEXT-4, include/rcm_cpu.h): plain C++17 + std::thread."""
    hdr = os.path.join(HERE, "..", "include", "rcm_cpu.h")
    if (not force and os.path.exists(CPU_LIB)
            and os.path.getmtime(CPU_LIB) >= max(os.path.getmtime(CPU_SRC), os.path.getmtime(hdr))):
        return CPU_LIB
    tmp = CPU_LIB + f".tmp{os.getpid()}"
    subprocess.check_call([CXX, "-O3", "-std=c++17", "-shared", "-fPIC", "-pthread", "-o", tmp, CPU_SRC])
    os.replace(tmp, CPU_LIB)
    return CPU_LIB


if __name__ == "__main__":
    print(build_cpu(force="--force" in sys.argv))
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
