"""ctypes binding of the host CPU-BATCH (``libcpubatch.so``, include/rcm_cpu.h):
the paper's batch-based RCM run by std::thread workers (SURVEY.md §8(f) NEXT-4,
P:L863-865).  A comparison implementation on the host -- never a fallback of the
GPU path, which does not import this module."""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libcpubatch.so")
_lib = None


class rcm_cpu_stats_t(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "batches_executed", "batches_empty", "rediscover_early", "rediscover_late",
        "candidates_removed", "chains")]


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"libcpubatch.so not built ({LIB_PATH}); run __graft_entry__.build()")
        lib = ctypes.CDLL(LIB_PATH)
        p32 = ctypes.POINTER(ctypes.c_int32)
        lib.rcm_cpu_batch.argtypes = [ctypes.c_int32, p32, p32, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                      ctypes.c_int32, ctypes.c_int32, p32, ctypes.POINTER(rcm_cpu_stats_t)]
        lib.rcm_cpu_batch.restype = ctypes.c_int
        _lib = lib
    return _lib


def rcm_cpu_batch(row_ptr, col_idx, mode: int = 1, start: int = 0, threads: int = 0,
                  batch_nodes: int = 0, temp_elems: int = 0, with_stats: bool = False):
    """perm (new -> old) of the CSR graph (host int32 arrays), computed by CPU-BATCH."""
    lib = _load()
    rp = np.ascontiguousarray(row_ptr, dtype=np.int32)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    n = len(rp) - 1
    perm = np.empty(n, dtype=np.int32)
    st = rcm_cpu_stats_t()
    p32 = ctypes.POINTER(ctypes.c_int32)
    rc = lib.rcm_cpu_batch(n, rp.ctypes.data_as(p32), ci.ctypes.data_as(p32) if len(ci) else None,
                           mode, start, threads, batch_nodes, temp_elems, perm.ctypes.data_as(p32),
                           ctypes.byref(st))
    if rc != 0:
        raise RuntimeError(f"rcm_cpu_batch failed with status {rc}")
    if with_stats:
        return perm, {n: int(getattr(st, n)) for n, _ in st._fields_}
    return perm
