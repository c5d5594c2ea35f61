"""Build librcm.so (sm_100a) in-tree with nvcc.  No torch at build time."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "librcm.so")
SOURCES = ["rcm.cu", "k_main_inst.cu", "k_solo.cu", "k_solo_sm.cu", "k_probe.cu"]
HEADERS = ["rcm_device.cuh", "rcm_batch.cuh", "rcm_workers.cuh", "rcm_lookback.cuh", "rcm_components.cuh",
           "rcm_leveled.cuh", "rcm_main.cuh", "rcm_solo.cuh"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = [*ARCH, "-O3", "-lineinfo", "-std=c++17", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC,-O2",
         "-Xptxas", "-warn-spills"]
# one translation unit per persistent-kernel variant (compiled in parallel):
# (min blocks per SM, multi-batch execution)
KMAIN_VARIANTS = [(2, 0), (1, 0), (2, 1), (1, 1), (2, 2), (1, 2)]   # (blocks per SM, 0 chain / 1 multi-batch / 2 leveled)
BUILD_DIR = os.path.join(HERE, "..", "build", "obj")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(HERE, "..", "include", "rcm.h"))
    deps.append(os.path.abspath(__file__))
    return any(os.path.getmtime(d) > t for d in deps if os.path.exists(d))


def _extra_defines() -> list:
    extra = [f"-DRCM_THREADS={os.environ['RCM_THREADS']}"] if os.environ.get("RCM_THREADS") else []
    if os.environ.get("RCM_DISC_U"):
        extra.append(f"-DRCM_DISC_U={os.environ['RCM_DISC_U']}")
    if os.environ.get("RCM_TRACE"):
        extra.append("-DRCM_TRACE")
    for k in ("RCM_SOLO_U", "RCM_SOLO_Q", "RCM_SOLO_NT", "RCM_SOLO_MINB", "RCM_SOLO_PEND", "RCM_SOLO_PIPE", "RCM_DQ_SLEEP_MAX", "RCM_LB_SLEEP_MAX", "RCM_CC_SAMPLE"):   # solo-path variants (sweeps)
        if os.environ.get(k):
            extra.append(f"-D{k}={os.environ[k]}")
    return extra


def build(force: bool = False, verbose: bool = False, out: str | None = None) -> str:
    """nvcc -c of every translation unit in parallel, then one -shared link.
    `out`: an alternative library path (variant builds for A/B sweeps, loaded
    with RCM_LIB=...; objects then go to a private directory)."""
    lib = out or LIB
    if not force and not out and not _stale():
        return LIB
    bdir = BUILD_DIR if not out else os.path.join(BUILD_DIR, os.path.basename(out) + ".obj")
    os.makedirs(bdir, exist_ok=True)
    extra = _extra_defines()
    if verbose:
        extra = ["-Xptxas=-v", *extra]
    jobs = [(os.path.join(bdir, "rcm.o"), [os.path.join(CSRC, "rcm.cu")]),
            (os.path.join(bdir, "k_solo.o"), [os.path.join(CSRC, "k_solo.cu")]),
            (os.path.join(bdir, "k_solo_sm.o"), [os.path.join(CSRC, "k_solo_sm.cu")]),
            (os.path.join(bdir, "k_probe.o"), [os.path.join(CSRC, "k_probe.cu")])]
    for bps, mb in KMAIN_VARIANTS:
        jobs.append((os.path.join(bdir, f"k_main_{bps}_{mb}.o"),
                     [f"-DRCM_KBPS={bps}", f"-DRCM_KMB={mb}", os.path.join(CSRC, "k_main_inst.cu")]))
    procs = []
    for obj, args in jobs:
        cmd = [NVCC, *FLAGS, *extra, "-c", "-o", obj + f".tmp{os.getpid()}", *args]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        procs.append((obj, subprocess.Popen(cmd)))
    bad = [obj for obj, p in procs if p.wait() != 0]
    if bad:
        raise subprocess.CalledProcessError(1, f"nvcc failed for {bad}")
    for obj, _ in procs:
        os.replace(obj + f".tmp{os.getpid()}", obj)
    tmp = lib + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-cudart", "static", "-Xcompiler", "-fPIC", "-Xlinker", "--no-undefined", "-o", tmp,
                           *[obj for obj, _ in jobs]])
    os.replace(tmp, lib)
    return lib


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
    outs = [a[len("--out="):] for a in sys.argv if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, out=outs[0] if outs else None))
