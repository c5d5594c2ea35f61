"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no traversal, no sorting by
valence, no ordering): it only builds symmetric CSR matrices of the shapes the
paper's workloads have (Table I: FEM meshes, structured grids,
power-law graphs), exactly as DESIGN.md "Input recipe" states.  Both the oracle
tests and the GPU tests/bench call it; it imports neither side.

Conventions: ``row_ptr`` int32 (n+1), ``col_idx`` int32, every row's columns
sorted ascending and unique, pattern structurally symmetric.  ``diag=True``
stores the diagonal (Laplacian/FEM pattern), ``diag=False`` is pure adjacency.
Relabelling uses a counter-based Feistel permutation (``randperm``) so that a
device generator can reproduce it bit-exactly without a shared RNG stream.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


# --------------------------------------------------------------------------- CSR
@dataclass
class CSR:
    n: int
    row_ptr: np.ndarray
    col_idx: np.ndarray
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr.astype(np.int64)).astype(np.int32)


def csr_from_pairs(n: int, src, dst, diag: bool = False, symmetrize: bool = True) -> CSR:
    """CSR of the pattern {(src,dst)} (+ transposes if symmetrize, + diagonal if
    diag) with self-loops of the input dropped, duplicates removed, columns sorted."""
    src = np.asarray(src, dtype=np.int64).ravel()
    dst = np.asarray(dst, dtype=np.int64).ravel()
    keep = src != dst
    src, dst = src[keep], dst[keep]
    if symmetrize:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
    if diag:
        ar = np.arange(n, dtype=np.int64)
        src, dst = np.concatenate([src, ar]), np.concatenate([dst, ar])
    key = np.sort(src * n + dst)
    if key.size:
        key = key[np.concatenate([[True], key[1:] != key[:-1]])]
    rows = key // n
    cols = (key - rows * n).astype(np.int32)
    counts = np.bincount(rows, minlength=n)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    assert row_ptr[-1] < 2**31, "int32 CSR overflow"
    return CSR(n, row_ptr.astype(np.int32), cols)


def relabel(g: CSR, perm_new_of_old: np.ndarray) -> CSR:
    """Rename node v to perm_new_of_old[v]; rebuild with sorted columns."""
    n = g.n
    p = np.asarray(perm_new_of_old, dtype=np.int64)
    deg = np.diff(g.row_ptr.astype(np.int64))
    src = np.repeat(p, deg)
    dst = p[g.col_idx.astype(np.int64)]
    key = np.sort(src * n + dst)
    rows = key // n
    cols = (key - rows * n).astype(np.int32)
    counts = np.bincount(rows, minlength=n)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return CSR(n, row_ptr.astype(np.int32), cols, dict(g.meta))


def disjoint_union(graphs) -> CSR:
    rps, cis, off, noff = [np.zeros(1, np.int64)], [], 0, 0
    for g in graphs:
        rps.append(g.row_ptr[1:].astype(np.int64) + noff)
        cis.append(g.col_idx.astype(np.int64) + off)
        off += g.n
        noff += g.nnz
    rp = np.concatenate(rps).astype(np.int32)
    ci = np.concatenate(cis).astype(np.int32) if cis else np.zeros(0, np.int32)
    return CSR(off, rp, ci)


# ------------------------------------------------- counter-based permutation
def _mix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = x.astype(np.uint64)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def feistel_bits(n: int) -> int:
    b = max(2, (max(n, 2) - 1).bit_length())
    return b + (b & 1)


def randperm(n: int, seed: int) -> np.ndarray:
    """Pseudo-random permutation of range(n): a 4-round balanced Feistel network
    over 2^(2h) >= n keyed by splitmix64(seed, round), cycle-walked into [0, n).
    Returns perm with perm[i] = image of i (a bijection of range(n))."""
    if n <= 1:
        return np.zeros(n, dtype=np.int64)
    bits = feistel_bits(n)
    h = bits // 2
    mask = np.uint64((1 << h) - 1)
    keys = [_mix64(np.array([(seed * 4 + r + 1) * 0x9E3779B97F4A7C15 & 0xFFFFFFFFFFFFFFFF],
                            dtype=np.uint64))[0] for r in range(4)]

    def enc(x):
        left = (x >> np.uint64(h)) & mask
        right = x & mask
        with np.errstate(over="ignore"):
            for r in range(4):
                f = _mix64(right ^ keys[r]) & mask
                left, right = right, left ^ f
        return (left << np.uint64(h)) | right

    x = np.arange(n, dtype=np.uint64)
    y = enc(x)
    bad = y >= np.uint64(n)
    while bad.any():
        y[bad] = enc(y[bad])
        bad = y >= np.uint64(n)
    return y.astype(np.int64)


# ------------------------------------------------------------ tiny families
def path(n: int, diag: bool = False) -> CSR:
    a = np.arange(n - 1)
    return csr_from_pairs(n, a, a + 1, diag)


def cycle(n: int, diag: bool = False) -> CSR:
    a = np.arange(n)
    return csr_from_pairs(n, a, (a + 1) % n, diag)


def star(m: int, diag: bool = False) -> CSR:
    """K_{1,m}, centre 0, leaves 1..m."""
    leaves = np.arange(1, m + 1)
    return csr_from_pairs(m + 1, np.zeros(m, np.int64), leaves, diag)


def complete(n: int, diag: bool = False) -> CSR:
    i, j = np.triu_indices(n, 1)
    return csr_from_pairs(n, i, j, diag)


def binary_tree(n: int, diag: bool = False) -> CSR:
    c = np.arange(1, n)
    return csr_from_pairs(n, (c - 1) // 2, c, diag)


def gnp(n: int, p: float, seed: int, diag: bool = False) -> CSR:
    rng = np.random.default_rng(seed)
    i, j = np.triu_indices(n, 1)
    keep = rng.random(i.size) < p
    return csr_from_pairs(n, i[keep], j[keep], diag)


def grid2d(w: int, h: int, diag: bool = False) -> CSR:
    """w x h 5-point grid, id = y*w + x (row-major)."""
    ids = np.arange(w * h).reshape(h, w)
    src = np.concatenate([ids[:, :-1].ravel(), ids[:-1, :].ravel()])
    dst = np.concatenate([ids[:, 1:].ravel(), ids[1:, :].ravel()])
    return csr_from_pairs(w * h, src, dst, diag)


def grid3d_27(nx: int, ny: int, nz: int, diag: bool = True) -> CSR:
    """nx x ny x nz 27-point stencil (all 26 Chebyshev neighbours), id = (z*ny + y)*nx + x.
    Built row by row with sorted columns directly (no global sort)."""
    n = nx * ny * nz
    x = np.arange(nx)
    y = np.arange(ny)
    z = np.arange(nz)
    cnt = lambda a, m: 1 + (a > 0) + (a < m - 1)  # noqa: E731
    deg = (cnt(z, nz)[:, None, None] * cnt(y, ny)[None, :, None] * cnt(x, nx)[None, None, :]).ravel()
    if not diag:
        deg = deg - 1
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(deg, out=row_ptr[1:])
    col = np.empty(int(row_ptr[-1]), dtype=np.int32)
    zz, yy, xx = np.meshgrid(z, y, x, indexing="ij")
    zz, yy, xx = zz.ravel(), yy.ravel(), xx.ravel()
    fill = row_ptr[:-1].copy()
    # offsets in increasing id order: dz major, then dy, then dx
    for dz in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dx in (-1, 0, 1):
                if not diag and dz == 0 and dy == 0 and dx == 0:
                    continue
                ok = ((xx + dx >= 0) & (xx + dx < nx) & (yy + dy >= 0) & (yy + dy < ny)
                      & (zz + dz >= 0) & (zz + dz < nz))
                rows = np.nonzero(ok)[0]
                col[fill[rows]] = rows + (dz * ny + dy) * nx + dx
                fill[rows] += 1
    assert np.array_equal(fill, row_ptr[1:])
    return CSR(n, row_ptr.astype(np.int32), col)


# ----------------------------------------------------------- paper workloads
def rmat_pairs(scale: int, edge_factor: int, seed: int, abcd=(0.57, 0.19, 0.19, 0.05)):
    """Graph500-style R-MAT edge samples (directed, may repeat / self-loop)."""
    rng = np.random.default_rng(seed)
    m = edge_factor << scale
    a, b, c, _ = abcd
    src = np.zeros(m, dtype=np.int64)
    dst = np.zeros(m, dtype=np.int64)
    for lvl in range(scale):
        r = rng.random(m, dtype=np.float32)
        bit_s = r >= np.float32(a + b)                      # quadrants c, d: row bit set
        bit_d = ((r >= np.float32(a)) & (r < np.float32(a + b))) | (r >= np.float32(a + b + c))
        src |= bit_s.astype(np.int64) << lvl
        dst |= bit_d.astype(np.int64) << lvl
    return src, dst


def rgg_expected_degree(n: int, r: float) -> float:
    """Expected degree in a unit-cube RGG with boundary effects (r <= 1/2):
    (n-1) * integral over |d|<r of prod_i (1-|d_i|)
      = (n-1) * (4/3 pi r^3 - 3/2 pi r^4 + 8/5 r^5 - 1/6 r^6)."""
    return (n - 1) * (4 / 3 * math.pi * r**3 - 1.5 * math.pi * r**4 + 1.6 * r**5 - r**6 / 6)


def rgg_radius(n: int, target_mean_deg: float) -> float:
    """Radius with expected mean degree == target (bisection on the closed form)."""
    lo, hi = 0.0, 0.5
    for _ in range(100):
        mid = 0.5 * (lo + hi)
        if rgg_expected_degree(n, mid) < target_mean_deg:
            lo = mid
        else:
            hi = mid
    return 0.5 * (lo + hi)


def rgg3d(n: int, mean_deg: float, seed: int) -> CSR:
    """Random geometric graph: n uniform points in [0,1)^3, edge iff distance < r,
    r tuned so the mean degree is mean_deg; ids in generation order; no diagonal."""
    from scipy.spatial import cKDTree
    pts = np.random.default_rng(seed).random((n, 3))
    r = rgg_radius(n, mean_deg)
    pairs = cKDTree(pts).query_pairs(r, output_type="ndarray")
    g = csr_from_pairs(n, pairs[:, 0], pairs[:, 1], diag=False)
    g.meta.update(radius=r, mean_deg=g.nnz / n)
    return g


def config_graph(cfg: int, scale: str = "full") -> tuple[CSR, int, int]:
    """(graph, start mode, start) for BASELINE.json configs 1..4.
    start mode: 0 FIXED, 1 MIN_DEGREE.  ``scale='small'`` gives the CI-sized twin."""
    small = scale == "small"
    if cfg == 1:   # 2D 5-point Laplacian 64x64, diagonal, shuffled labels, start 0
        w = 64 if not small else 16
        g = relabel(grid2d(w, w, diag=True), randperm(w * w, 1))
        g.meta.update(name=f"grid2d_5pt_{w}x{w}")
        return g, 0, 0
    if cfg == 2:   # 3D 27-point FEM-like grid 100^3, diagonal, relabelled (seed 2)
        a = 100 if not small else 20
        g = relabel(grid3d_27(a, a, a, diag=True), randperm(a ** 3, 2))
        g.meta.update(name=f"grid3d_27pt_{a}^3")
        return g, 1, 0
    if cfg == 3:   # tetrahedral-mesh-shaped RGG, 4M nodes, mean degree 14
        n = 4_000_000 if not small else 60_000
        g = rgg3d(n, 14.0, 3)
        g.meta.update(name=f"rgg3d_{n}")
        return g, 1, 0
    if cfg == 4:   # R-MAT 2^22, 8 * 2^22 samples, symmetrised, relabelled (seed 40)
        sc = 22 if not small else 14
        s, d = rmat_pairs(sc, 8, 4)
        g = csr_from_pairs(1 << sc, s, d, diag=False)
        g = relabel(g, randperm(1 << sc, 40))
        g.meta.update(name=f"rmat_s{sc}")
        return g, 1, 0
    raise ValueError(cfg)


# --------------------------------------------------------- config 5 (batch)
def c5_sizes(num: int = 8192, seed: int = 5, lo: float = 1e3, hi: float = 1e5) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return np.round(np.exp(rng.uniform(math.log(lo), math.log(hi), num))).astype(np.int64)


def c5_dims(k: int, N: int):
    """Even k: 2D 5-point w x h; odd k: 3D 27-point near-cube a x a x c."""
    if k % 2 == 0:
        w = max(2, int(round(math.sqrt(N))))
        h = max(2, int(round(N / w)))
        return (w, h)
    a = max(2, int(round(N ** (1 / 3))))
    c = max(2, int(round(N / (a * a))))
    return (a, a, c)


def c5_matrix(k: int, N: int) -> CSR:
    dims = c5_dims(k, N)
    g = grid2d(*dims, diag=True) if len(dims) == 2 else grid3d_27(*dims, diag=True)
    return relabel(g, randperm(g.n, 50000 + k))


@dataclass
class Batch:
    node_off: np.ndarray     # int64 (num+1)
    nnz_off: np.ndarray      # int64 (num+1)
    row_ptr_local: np.ndarray  # int32, per matrix n_k+1 entries, concatenated
    col_idx_local: np.ndarray  # int32 local ids
    dims: list


def c5_batch(num: int = 8192, seed: int = 5, lo: float = 1e3, hi: float = 1e5) -> Batch:
    sizes = c5_sizes(num, seed, lo, hi)
    mats = [c5_matrix(k, int(N)) for k, N in enumerate(sizes)]
    return batch_of(mats, [c5_dims(k, int(N)) for k, N in enumerate(sizes)])


def batch_of(mats, dims=None) -> Batch:
    node_off = np.zeros(len(mats) + 1, np.int64)
    nnz_off = np.zeros(len(mats) + 1, np.int64)
    node_off[1:] = np.cumsum([m.n for m in mats])
    nnz_off[1:] = np.cumsum([m.nnz for m in mats])
    rp = np.concatenate([m.row_ptr for m in mats]).astype(np.int32)
    ci = np.concatenate([m.col_idx for m in mats]).astype(np.int32)
    return Batch(node_off, nnz_off, rp, ci, dims or [None] * len(mats))
