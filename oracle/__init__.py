"""Serial RCM oracle -- TEST INFRASTRUCTURE ONLY.

A plain CPU implementation of what the hot path computes, written from the paper
(Mlakar et al., IPDPS'21; ``P:L<n>`` = /root/reference/PAPER.md line n):

* ``rcm``        -- Alg. 1 Sequential RCM + the C-6 component rule
* ``gl``         -- pseudo-peripheral node finder (sec. III-d)
* ``bfs_levels`` -- plain BFS levels used by ``gl``
* ``degree``     -- valence v = r[n+1] - r[n]
* ``bandwidth``  -- max |pos(i) - pos(j)| over stored off-diagonals (C-15)

The arithmetic lives in ``rcm_oracle.c`` (plain C, single thread); this module
only marshals numpy arrays.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` leg may import it.  It
shares no code with ``paper_conf_ipps_mlakarwps21_b200`` and never imports it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "rcm_oracle.c")
_LIB_PATH = os.path.join(_HERE, "librcm_oracle.so")
_lib = None
_lock = threading.Lock()

FIXED, MIN_DEGREE, PSEUDO_PERIPHERAL = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile rcm_oracle.c with gcc (building the checker is not using it)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=native", "-std=c99", "-Wall", "-Wextra",
                               "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            i32p = ctypes.POINTER(ctypes.c_int32)
            lib.oracle_degree.argtypes = [ctypes.c_int32, i32p, i32p]
            lib.oracle_bfs_levels.argtypes = [ctypes.c_int32, i32p, i32p, ctypes.c_int32, i32p]
            lib.oracle_bfs_levels.restype = ctypes.c_int32
            lib.oracle_gl.argtypes = [ctypes.c_int32, i32p, i32p, ctypes.c_int32]
            lib.oracle_gl.restype = ctypes.c_int32
            lib.oracle_rcm.argtypes = [ctypes.c_int32, i32p, i32p, ctypes.c_int32, ctypes.c_int32, i32p, i32p]
            lib.oracle_rcm.restype = ctypes.c_int
            lib.oracle_bandwidth.argtypes = [ctypes.c_int32, i32p, i32p, i32p]
            lib.oracle_bandwidth.restype = ctypes.c_int64
            _lib = lib
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)) if a is not None else None


def _csr(row_ptr, col_idx):
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int32)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    if col_idx.size == 0:
        col_idx = np.zeros(1, dtype=np.int32)
    return row_ptr, col_idx


def degree(row_ptr) -> np.ndarray:
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int32)
    n = row_ptr.size - 1
    out = np.empty(n, dtype=np.int32)
    assert _load().oracle_degree(n, _p(row_ptr), _p(out)) == 0
    return out


def bfs_levels(row_ptr, col_idx, root: int):
    """(level array with -1 for unreachable, number of levels)."""
    row_ptr, col_idx = _csr(row_ptr, col_idx)
    n = row_ptr.size - 1
    lev = np.empty(n, dtype=np.int32)
    nlev = _load().oracle_bfs_levels(n, _p(row_ptr), _p(col_idx), int(root), _p(lev))
    return lev, int(nlev)


def gl(row_ptr, col_idx, root: int) -> int:
    row_ptr, col_idx = _csr(row_ptr, col_idx)
    n = row_ptr.size - 1
    return int(_load().oracle_gl(n, _p(row_ptr), _p(col_idx), int(root)))


def rcm(row_ptr, col_idx, mode: int = MIN_DEGREE, start: int = 0, return_order: bool = False):
    """Serial RCM permutation perm (new -> old), optionally also the CM order o."""
    row_ptr, col_idx = _csr(row_ptr, col_idx)
    n = row_ptr.size - 1
    perm = np.empty(max(n, 1), dtype=np.int32)
    o = np.empty(max(n, 1), dtype=np.int32) if return_order else None
    st = _load().oracle_rcm(n, _p(row_ptr), _p(col_idx), int(mode), int(start), _p(perm), _p(o))
    if st != 0:
        raise ValueError(f"oracle_rcm failed with status {st}")
    perm = perm[:n]
    return (perm, o[:n]) if return_order else perm


def rcm_batched(node_off, nnz_off, row_ptr_local, col_idx_local, mode: int = MIN_DEGREE,
                starts=None, threads: int = 1, mats=None):
    """Per-matrix serial RCM over a concatenated batch (same layout as
    rcm_reorder_batched).  Returns perm_local (concatenated local new->old).
    ``mats`` restricts the work to a subset (others left as -1).  ``threads`` > 1
    runs independent matrices on a thread pool (ctypes releases the GIL)."""
    node_off = np.asarray(node_off, dtype=np.int64)
    nnz_off = np.asarray(nnz_off, dtype=np.int64)
    num = node_off.size - 1
    out = np.full(int(node_off[-1]), -1, dtype=np.int32)
    idx = range(num) if mats is None else list(mats)

    def one(k):
        a, b = int(node_off[k]), int(node_off[k + 1])
        rp = row_ptr_local[a + k: b + k + 1]
        ci = col_idx_local[int(nnz_off[k]): int(nnz_off[k + 1])]
        s = 0 if starts is None else int(starts[k])
        out[a:b] = rcm(rp, ci, mode, s)

    if threads <= 1:
        for k in idx:
            one(k)
    else:
        from concurrent.futures import ThreadPoolExecutor
        with ThreadPoolExecutor(threads) as ex:
            list(ex.map(one, idx))
    return out


def bandwidth(row_ptr, col_idx, perm=None) -> int:
    row_ptr, col_idx = _csr(row_ptr, col_idx)
    n = row_ptr.size - 1
    perm = None if perm is None else np.ascontiguousarray(perm, dtype=np.int32)
    return int(_load().oracle_bandwidth(n, _p(row_ptr), _p(col_idx), _p(perm)))
