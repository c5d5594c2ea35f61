"""Generator checks: determinism, symmetry, sorted unique columns, nnz formulas."""
import numpy as np
import pytest

import synth


def _check_csr(g, diag=None):
    rp, ci = g.row_ptr.astype(np.int64), g.col_idx.astype(np.int64)
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0) and rp[-1] == ci.size
    assert ci.size == 0 or (ci.min() >= 0 and ci.max() < g.n)
    rows = np.repeat(np.arange(g.n), np.diff(rp))
    # sorted, unique within rows
    same_row = rows[1:] == rows[:-1]
    assert np.all(ci[1:][same_row] > ci[:-1][same_row])
    # symmetric pattern
    k1 = np.sort(rows * g.n + ci)
    k2 = np.sort(ci * g.n + rows)
    assert np.array_equal(k1, k2)
    if diag is not None:
        has = np.zeros(g.n, bool)
        has[rows[rows == ci]] = True
        assert has.all() if diag else not has.any()


def test_randperm_is_bijection_and_deterministic():
    for n in [1, 2, 3, 17, 1000, 4096, 12345]:
        p = synth.randperm(n, 7)
        assert np.array_equal(np.sort(p), np.arange(n))
        assert np.array_equal(p, synth.randperm(n, 7))
    assert not np.array_equal(synth.randperm(1000, 1), synth.randperm(1000, 2))


@pytest.mark.parametrize("w,h", [(2, 2), (5, 3), (64, 64)])
def test_grid2d(w, h):
    g = synth.grid2d(w, h, diag=True)
    _check_csr(g, diag=True)
    assert g.nnz == w * h + 2 * ((w - 1) * h + w * (h - 1))


@pytest.mark.parametrize("dims", [(2, 2, 2), (3, 4, 5), (10, 10, 10)])
def test_grid3d_27(dims):
    g = synth.grid3d_27(*dims, diag=True)
    _check_csr(g, diag=True)
    c = lambda m: 3 * m - 2  # noqa: E731  (pairs |i-j|<=1 in 1D)
    assert g.nnz == c(dims[0]) * c(dims[1]) * c(dims[2])
    g0 = synth.grid3d_27(*dims, diag=False)
    _check_csr(g0, diag=False)


def test_config_small_twins_are_valid():
    for cfg, diag in [(1, True), (2, True), (3, False), (4, False)]:
        g, mode, s = synth.config_graph(cfg, "small")
        _check_csr(g, diag=diag if cfg != 4 else None)
        g2, _, _ = synth.config_graph(cfg, "small")
        assert np.array_equal(g.row_ptr, g2.row_ptr) and np.array_equal(g.col_idx, g2.col_idx)


def test_config1_shape():
    g, mode, s = synth.config_graph(1)
    assert (g.n, g.nnz, mode, s) == (4096, 20224, 0, 0)
    assert set(np.unique(np.diff(g.row_ptr))) == {3, 4, 5}


def test_rgg_closed_form_radius():
    # closed form expected degree vs brute-force count on a small instance
    n = 20000
    r = synth.rgg_radius(n, 14.0)
    assert abs(synth.rgg_expected_degree(n, r) - 14.0) < 1e-6
    g = synth.rgg3d(n, 14.0, 5)
    assert abs(g.nnz / n - 14.0) < 0.5


def test_c5_batch_small():
    b = synth.c5_batch(num=6, seed=5, lo=50, hi=300)
    assert b.node_off.size == 7 and b.nnz_off[-1] == b.col_idx_local.size
    for k in range(6):
        a, e = b.node_off[k], b.node_off[k + 1]
        rp = b.row_ptr_local[a + k:e + k + 1]
        ci = b.col_idx_local[b.nnz_off[k]:b.nnz_off[k + 1]]
        _check_csr(synth.CSR(int(e - a), rp, ci), diag=True)
