"""Pins for the serial RCM oracle, CPU only.

Each test pins the oracle against something other than itself: the independent
CM-order verifier (tests/verifier.py), exhaustive brute force, closed forms,
scipy's RCM, and the paper's printed ecology1 bandwidth (tests/golden/).
"""
from __future__ import annotations

import itertools
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import connected_components, reverse_cuthill_mckee, shortest_path

import oracle
import synth
from verifier import bandwidth_py, gl_py, verify, verify_small

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _sp(g):
    return sp.csr_matrix((np.ones(g.nnz), g.col_idx, g.row_ptr), shape=(g.n, g.n))


def _graph_from_edges(n, edges, diag=False):
    if not edges:
        src = dst = np.zeros(0, np.int64)
    else:
        src, dst = np.array(edges).T
    return synth.csr_from_pairs(n, src, dst, diag)


# ----------------------------------------------------------------- P7 degree
def test_degree_is_row_length():
    g = synth.gnp(50, 0.1, 3, diag=True)
    assert np.array_equal(oracle.degree(g.row_ptr), np.diff(g.row_ptr))


# ------------------------------------------------------------ P3 closed forms
@pytest.mark.parametrize("n", [2, 3, 7, 20])
@pytest.mark.parametrize("diag", [False, True])
def test_path_from_end_is_identity(n, diag):
    g = synth.path(n, diag)
    perm, o = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0, return_order=True)
    assert np.array_equal(o, np.arange(n))
    assert np.array_equal(perm, np.arange(n)[::-1])
    assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) == 1


def _path_interior_closed_form(n, j):
    deg = lambda v: 1 if v in (0, n - 1) else 2  # noqa: E731
    left_first = (deg(j - 1), j - 1) < (deg(j + 1), j + 1)
    o = [j]
    for d in range(1, n):
        lv = [v for v in ((j - d, j + d) if left_first else (j + d, j - d)) if 0 <= v < n]
        o += lv
    return o


@pytest.mark.parametrize("n,j", [(9, 4), (9, 1), (9, 7), (10, 2), (5, 3), (12, 9)])
def test_path_from_interior(n, j):
    g = synth.path(n)
    _, o = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, j, return_order=True)
    assert list(o) == _path_interior_closed_form(n, j)


@pytest.mark.parametrize("n", [3, 4, 9, 10])
def test_cycle_from_zero(n):
    g = synth.cycle(n)
    _, o = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0, return_order=True)
    exp = [0]
    for d in range(1, n):
        for v in (d, n - d):
            if v not in exp:
                exp.append(v)
    assert list(o) == exp[:n]
    assert oracle.bandwidth(g.row_ptr, g.col_idx, oracle.rcm(g.row_ptr, g.col_idx, 0, 0)) == 2


@pytest.mark.parametrize("m", [1, 4, 9])
def test_star(m):
    g = synth.star(m)
    _, o = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0, return_order=True)
    assert list(o) == list(range(m + 1))
    for j in range(1, m + 1):
        _, o = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, j, return_order=True)
        assert list(o) == [j, 0] + [v for v in range(1, m + 1) if v != j]


@pytest.mark.parametrize("n,s", [(5, 0), (6, 3), (8, 7)])
def test_complete(n, s):
    g = synth.complete(n)
    perm, o = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, s, return_order=True)
    assert list(o) == [s] + [v for v in range(n) if v != s]
    assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) == n - 1


def _grid_closed_form(w, h):
    o = []
    for d in range(w + h - 1):
        for x in range(min(d, w - 1), max(0, d - h + 1) - 1, -1):
            o.append((d - x) * w + x)
    return o


@pytest.mark.parametrize("w,h", [(2, 2), (3, 5), (5, 3), (7, 7), (8, 3), (3, 8), (13, 40), (40, 13)])
@pytest.mark.parametrize("diag", [False, True])
def test_grid_antidiagonals(w, h, diag):
    g = synth.grid2d(w, h, diag)
    perm, o = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0, return_order=True)
    assert list(o) == _grid_closed_form(w, h)
    assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) == (w if w <= h else h + 1)


# ----------------------------------------------- P5 paper value (ecology1 twin)
def test_ecology1_twin_bandwidth():
    fx = dict(l.strip().split("=") for l in open(os.path.join(GOLDEN, "ecology1_bandwidth.txt"))
              if "=" in l and not l.startswith("#"))
    w = int(round(int(fx["n"]) ** 0.5))
    g = synth.grid2d(w, w, diag=True)
    assert g.nnz == 4_996_000                                   # Table I "5.0M"
    assert oracle.bandwidth(g.row_ptr, g.col_idx) == int(fx["init_bw"])
    perm = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0)
    assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) == int(fx["reord_bw"])
    assert bandwidth_py(g.row_ptr, g.col_idx, perm) == int(fx["reord_bw"])


# -------------------------------------------- P1 verifier on assorted graphs
def _assorted():
    gs = [synth.gnp(60, 0.05, s) for s in range(6)]
    gs += [synth.gnp(40, 0.2, 10 + s, diag=True) for s in range(3)]
    gs += [synth.binary_tree(31), synth.grid2d(9, 6), synth.star(7), synth.cycle(11)]
    gs.append(synth.disjoint_union([synth.path(4), synth.star(3), synth.complete(4), synth.path(1)]))
    gs.append(synth.relabel(synth.grid3d_27(5, 4, 3), synth.randperm(60, 9)))
    return gs


@pytest.mark.parametrize("mode", [oracle.FIXED, oracle.MIN_DEGREE, oracle.PSEUDO_PERIPHERAL])
def test_oracle_passes_verifier(mode):
    for g in _assorted():
        for s in ([0, g.n // 2, g.n - 1] if mode == oracle.FIXED else [0]):
            perm = oracle.rcm(g.row_ptr, g.col_idx, mode, s)
            assert verify(g.row_ptr, g.col_idx, perm, mode, s) is None
            assert verify_small(g.row_ptr, g.col_idx, perm, mode, s) is None


def test_duplicates_and_self_loops_count_in_valence():
    # C-2 / C-8: duplicates and self loops count in the valence, are skipped as children.
    rp = np.array([0, 3, 6, 8, 10, 11], np.int32)
    ci = np.array([1, 2, 2,  0, 1, 3,  0, 0,  1, 4,  3], np.int32)  # node1 has a self loop, node2 dup 0
    perm, o = oracle.rcm(rp, ci, oracle.FIXED, 0, return_order=True)
    # children of 0: 1 (deg 3) and 2 (deg 2, row [0,0]) -> 2 first
    assert list(o[:3]) == [0, 2, 1]
    assert verify(rp, ci, perm, oracle.FIXED, 0) is None
    assert verify_small(rp, ci, perm, oracle.FIXED, 0) is None


def test_verifier_rejects_perturbations():
    g = synth.relabel(synth.grid2d(6, 5), synth.randperm(30, 4))
    perm = oracle.rcm(g.row_ptr, g.col_idx, oracle.MIN_DEGREE)
    rng = np.random.default_rng(0)
    rejected = 0
    for _ in range(50):
        p = perm.copy()
        i, j = rng.choice(g.n, 2, replace=False)
        p[i], p[j] = p[j], p[i]
        if verify(g.row_ptr, g.col_idx, p, 1) is not None:
            rejected += 1
            assert verify_small(g.row_ptr, g.col_idx, p, 1) is not None
    assert rejected == 50


# --------------------------------------------------- P2 exhaustive brute force
def _all_graphs(n):
    pairs = list(itertools.combinations(range(n), 2))
    for mask in range(1 << len(pairs)):
        yield [pairs[k] for k in range(len(pairs)) if mask >> k & 1]


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5])
def test_bruteforce_unique_and_equal(n):
    perms = list(itertools.permutations(range(n)))
    for edges in _all_graphs(n):
        g = _graph_from_edges(n, edges)
        rp, ci = g.row_ptr.tolist(), g.col_idx.tolist()
        for mode, s in [(1, 0)] + [(0, s) for s in range(n)]:
            ok = [p for p in perms if verify_small(rp, ci, p, mode, s) is None]
            assert len(ok) == 1, (edges, mode, s, ok)
            assert tuple(oracle.rcm(g.row_ptr, g.col_idx, mode, s)) == ok[0]


# ------------------------------------------------------- P4 scipy RCM (connected)
def _connected_samples():
    out = []
    for s in range(8):
        g = synth.gnp(80, 0.06, 100 + s)
        if connected_components(_sp(g))[0] == 1:
            out.append(g)
    out += [synth.relabel(synth.grid2d(12, 9, True), synth.randperm(108, 7)),
            synth.relabel(synth.grid3d_27(6, 5, 4, True), synth.randperm(120, 8)),
            synth.relabel(synth.binary_tree(63), synth.randperm(63, 5))]
    return out


def test_matches_scipy_rcm_on_connected_graphs():
    gs = _connected_samples()
    assert len(gs) >= 6
    for g in gs:
        sperm = reverse_cuthill_mckee(_sp(g), symmetric_mode=True)
        root = int(sperm[-1])
        perm = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, root)
        assert np.array_equal(perm, sperm)


# ------------------------------------- P6 bandwidth vs brute-force optimum
def _min_bw(g):
    n = g.n
    rows = np.repeat(np.arange(n), np.diff(g.row_ptr))
    cols = g.col_idx
    off = rows != cols
    rows, cols = rows[off], cols[off]
    best = n
    for p in itertools.permutations(range(n)):
        pos = np.empty(n, np.int64)
        pos[list(p)] = np.arange(n)
        best = min(best, int(np.abs(pos[rows] - pos[cols]).max()) if rows.size else 0)
    return best


@pytest.mark.parametrize("name,g,opt", [
    ("path7", synth.path(7), 1), ("cycle7", synth.cycle(7), 2), ("K6", synth.complete(6), 5),
])
def test_bandwidth_optimal_families(name, g, opt):
    assert _min_bw(g) == opt
    perm = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0)
    assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) == opt


def test_bandwidth_lower_bound_random_and_star_gap():
    for s in range(4):
        g = synth.gnp(7, 0.4, 200 + s)
        perm = oracle.rcm(g.row_ptr, g.col_idx, oracle.MIN_DEGREE)
        assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) >= _min_bw(g)
        assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) == bandwidth_py(g.row_ptr, g.col_idx, perm)
    g = synth.star(6)                                  # K_{1,6} from its centre: m > ceil(m/2)
    perm = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0)
    assert oracle.bandwidth(g.row_ptr, g.col_idx, perm) == 6 and _min_bw(g) == 3


# ------------------------------------------------------------------- P9 GL
@pytest.mark.parametrize("n", [2, 5, 30])
def test_gl_path_returns_far_end(n):
    g = synth.path(n)
    assert oracle.gl(g.row_ptr, g.col_idx, 0) == n - 1


@pytest.mark.parametrize("w,h", [(2, 2), (5, 3), (7, 7), (4, 11)])
def test_gl_grid_returns_opposite_corner(w, h):
    g = synth.grid2d(w, h)
    assert oracle.gl(g.row_ptr, g.col_idx, 0) == w * h - 1


def test_gl_properties_with_scipy_distances():
    for s in range(6):
        g = synth.gnp(40, 0.08, 300 + s)
        ncomp, lab = connected_components(_sp(g))
        r = int(np.argmin(np.diff(g.row_ptr) * (g.n + 1) + np.arange(g.n)))
        x = oracle.gl(g.row_ptr, g.col_idx, r)
        assert x == gl_py(g.row_ptr.tolist(), g.col_idx.tolist(), r)
        D = shortest_path(_sp(g), unweighted=True)
        ecc = lambda v: int(np.max(D[v][np.isfinite(D[v])]))  # noqa: E731
        assert lab[x] == lab[r]
        assert ecc(x) >= ecc(r)
        lev, nl = oracle.bfs_levels(g.row_ptr, g.col_idx, x)
        assert nl == ecc(x) + 1
        assert np.array_equal(np.where(lev >= 0, lev, -1),
                              np.where(np.isfinite(D[x]), D[x], -1).astype(np.int32))


# -------------------------------------------- P8 components (scipy partition)
def test_components_follow_min_key_rule():
    g = synth.disjoint_union([synth.grid2d(3, 3), synth.path(5), synth.star(4), synth.complete(3),
                              synth.path(1), synth.cycle(6)])
    g = synth.relabel(g, synth.randperm(g.n, 11))
    ncomp, lab = connected_components(_sp(g))
    for mode, s in [(oracle.MIN_DEGREE, 0), (oracle.FIXED, 7), (oracle.PSEUDO_PERIPHERAL, 0)]:
        perm = oracle.rcm(g.row_ptr, g.col_idx, mode, s)
        assert verify(g.row_ptr, g.col_idx, perm, mode, s) is None
        o = perm[::-1]
        # each component is one contiguous block of o
        seg_labels = lab[o]
        changes = np.count_nonzero(seg_labels[1:] != seg_labels[:-1])
        assert changes == ncomp - 1
