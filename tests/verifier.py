"""Independent Cuthill-McKee order verifier (SURVEY.md sec. 8(c) pin P1).

Written from the characterisation of the CM order, NOT from Alg. 1: it shares no
code with ``oracle/`` or with the CUDA path.  With o = reverse(perm) and
par(v) = the neighbour of v (v itself excluded) with the smallest position:

  V0  perm is a permutation of range(n)
  V1  a node is a root iff it has no earlier neighbour; every non-root's parent
      lies in the same root segment (segments are whole components)
  V2  over non-roots in o order, pos(par) is non-decreasing (FIFO / BFS order,
      Alg. 1 ln 6-7; Alg. 2's "lowest source")
  V3  equal parents => strictly increasing (valence, id) (Alg. 1 ln 14, C-1)
  V4  roots follow the start rule: FIXED first root = start; every other root
      is the minimum (valence, id) over the not-yet-placed suffix (C-6); with
      PSEUDO_PERIPHERAL that minimum refined by the GL finder (C-5)

Appendix B.2 of SURVEY.md shows V0-V4 determine the order uniquely.
Two implementations: ``verify_small`` (pure Python loops, for brute force) and
``verify`` (vectorised numpy, O(n + nnz), for large graphs).
"""
from __future__ import annotations

import numpy as np


def _deg(row_ptr):
    return np.diff(np.asarray(row_ptr, dtype=np.int64))


def gl_levels_py(row_ptr, col_idx, root):
    """Plain BFS levels (dict-free list version) for the GL check."""
    n = len(row_ptr) - 1
    lev = [-1] * n
    lev[root] = 0
    frontier = [root]
    nlev = 1
    while frontier:
        nxt = []
        for p in frontier:
            for e in range(row_ptr[p], row_ptr[p + 1]):
                c = int(col_idx[e])
                if lev[c] < 0:
                    lev[c] = lev[p] + 1
                    nxt.append(c)
        if nxt:
            nlev += 1
        frontier = nxt
    return lev, nlev


def gl_py(row_ptr, col_idx, r):
    """Pseudo-peripheral finder, independent re-statement."""
    deg = _deg(row_ptr)
    lev, nl = gl_levels_py(row_ptr, col_idx, r)
    while True:
        last = [v for v in range(len(lev)) if lev[v] == nl - 1]
        x = min(last, key=lambda v: (deg[v], v))
        lev_x, nl_x = gl_levels_py(row_ptr, col_idx, x)
        if nl_x > nl:
            lev, nl = lev_x, nl_x
            continue
        return x


def verify_small(row_ptr, col_idx, perm, mode=1, start=0):
    """Pure-Python V0-V4.  Returns None if valid, else a string naming the
    first violated condition."""
    n = len(row_ptr) - 1
    perm = [int(x) for x in perm]
    if sorted(perm) != list(range(n)):
        return "V0"
    o = perm[::-1]
    pos = [0] * n
    for i, v in enumerate(o):
        pos[v] = i
    deg = [int(row_ptr[v + 1] - row_ptr[v]) for v in range(n)]
    par = [None] * n
    for v in range(n):
        best = None
        for e in range(row_ptr[v], row_ptr[v + 1]):
            u = int(col_idx[e])
            if u != v and (best is None or pos[u] < best):
                best = pos[u]
        par[v] = best
    seg = [0] * n
    s = -1
    roots = []
    for i, v in enumerate(o):
        if par[v] is None or par[v] > i:
            s += 1
            roots.append(i)
        seg[i] = s
    if roots[0] != 0:
        return "V1"
    last_par = -1
    prev = None
    for i, v in enumerate(o):
        if par[v] is None or par[v] > i:
            continue
        if seg[par[v]] != seg[i]:
            return "V1"
        if par[v] < last_par:
            return "V2"
        if prev is not None and par[v] == last_par and (deg[prev], prev) >= (deg[v], v):
            return "V3"
        last_par, prev = par[v], v
    for k, i in enumerate(roots):
        v = o[i]
        if k == 0 and mode == 0:
            if v != start:
                return "V4"
            continue
        m = min(o[i:], key=lambda u: (deg[u], u))
        if mode == 2:
            m = gl_py(row_ptr, col_idx, m)
        if v != m:
            return "V4"
    return None


def verify(row_ptr, col_idx, perm, mode=1, start=0, check_gl=True, check_sort=True):
    """Vectorised V0-V4 (numpy, O(n + nnz) except V4 with mode 2 which runs a
    BFS per root).  Returns None if valid else the name of the failed check.
    check_sort=False skips V3: what is left (V0-V2, V4) characterises a BFS
    order with first-discovery parents, the output of RCM_FLAG_NO_SORT
    ("disable sorting ... BFS")."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col_idx = np.asarray(col_idx, dtype=np.int64)
    perm = np.asarray(perm, dtype=np.int64)
    n = row_ptr.size - 1
    if perm.size != n or not np.array_equal(np.sort(perm), np.arange(n)):
        return "V0"
    if n == 0:
        return None
    o = perm[::-1]
    pos = np.empty(n, np.int64)
    pos[o] = np.arange(n)
    deg = np.diff(row_ptr)
    rows = np.repeat(np.arange(n), deg)
    npos = np.where(col_idx != rows, pos[col_idx], np.int64(n))     # self loops ignored
    parpos = np.full(n, n, np.int64)
    np.minimum.at(parpos, rows, npos)
    # positions of o: is_root[i]
    pp = parpos[o]                                    # parent position of o[i]
    ipos = np.arange(n)
    is_root = pp > ipos
    if not is_root[0]:
        return "V1"
    seg = np.cumsum(is_root) - 1
    nr = ~is_root
    if np.any(seg[pp[nr]] != seg[ipos[nr]]):
        return "V1"
    ppn = pp[nr]
    if np.any(np.diff(ppn) < 0):
        return "V2"
    vn = o[nr]
    dn = deg[vn]
    same = ppn[1:] == ppn[:-1]
    kprev = dn[:-1] * (n + 1) + vn[:-1]
    knext = dn[1:] * (n + 1) + vn[1:]
    if check_sort and np.any(same & (kprev >= knext)):
        return "V3"
    # V4: suffix minimum of (deg, id) over o
    key = deg[o] * (n + 1) + o
    sufmin = np.minimum.accumulate(key[::-1])[::-1]
    ridx = np.nonzero(is_root)[0]
    for k, i in enumerate(ridx):
        v = int(o[i])
        if k == 0 and mode == 0:
            if v != start:
                return "V4"
            continue
        m = int(sufmin[i] % (n + 1))
        if mode == 2 and check_gl:
            m = gl_py(row_ptr, col_idx, m)
        if mode != 2 or check_gl:
            if v != m:
                return "V4"
    return None


def bandwidth_py(row_ptr, col_idx, perm=None):
    """C-15 bandwidth, vectorised, independent of the oracle."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col_idx = np.asarray(col_idx, dtype=np.int64)
    n = row_ptr.size - 1
    pos = np.arange(n) if perm is None else np.argsort(np.asarray(perm))
    rows = np.repeat(np.arange(n), np.diff(row_ptr))
    off = rows != col_idx
    if not off.any():
        return 0
    return int(np.abs(pos[rows[off]] - pos[col_idx[off]]).max())
