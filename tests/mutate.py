"""Test-side CSR mutators for the ABI's edge cases (include/rcm.h: duplicates
and self-loops are legal and count in the valence, sorted columns are not
required).  The generators in synth/ always emit sorted, duplicate-free rows,
so these mutations are the only way such inputs reach the GPU path.  No
arithmetic of the method lives here.  Every mutation keeps the pattern
structurally symmetric (a duplicate (u,c) is added together with (c,u))."""
from __future__ import annotations

import numpy as np

from synth import CSR


def _rebuild(n, rows, cols, rng, shuffle):
    order = np.lexsort((rng.random(rows.size) if shuffle else cols, rows))
    rows, cols = rows[order], cols[order]
    row_ptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(rows, minlength=n), out=row_ptr[1:])
    return CSR(n, row_ptr.astype(np.int32), cols.astype(np.int32))


def mutate(g: CSR, seed: int, dup: float = 0.0, loops: float = 0.0, shuffle: bool = False) -> CSR:
    """dup: fraction of stored off-diagonal entries (u,c) duplicated, with their
    transposes (some twice); loops: fraction of nodes given an extra diagonal
    entry (a second one if it already has one); shuffle: random column order
    inside every row."""
    rng = np.random.default_rng(seed)
    n = g.n
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(g.row_ptr.astype(np.int64)))
    cols = g.col_idx.astype(np.int64)
    add_r, add_c = [rows], [cols]
    if dup > 0:
        off = np.nonzero(rows != cols)[0]
        pick = off[rng.random(off.size) < dup]
        twice = pick[rng.random(pick.size) < 0.25]
        for p in (pick, twice):
            add_r += [rows[p], cols[p]]
            add_c += [cols[p], rows[p]]
    if loops > 0:
        v = np.nonzero(rng.random(n) < loops)[0]
        add_r.append(v)
        add_c.append(v)
    return _rebuild(n, np.concatenate(add_r), np.concatenate(add_c), rng, shuffle)


def unsorted(g: CSR, seed: int) -> CSR:
    return mutate(g, seed, shuffle=True)


ALL = {
    "dup": dict(dup=0.15),
    "loops": dict(loops=0.3),
    "shuffle": dict(shuffle=True),
    "all": dict(dup=0.1, loops=0.2, shuffle=True),
}
