"""GPU: the ABI's edge cases and error paths, through the C ABI, against the
oracle (bit-exact) or the independent verifier.

* duplicates, self-loops and unsorted rows (include/rcm.h: all legal; they count
  in the valence, C-2 / P:L209, and are skipped as children, C-8 / P:L204-205);
* PSEUDO_PERIPHERAL (GL start finder, C-5) on the full configs, and
  rcm_find_pseudo_peripheral against oracle.gl at full size;
* RCM_FLAG_NO_SORT emits a BFS order: V0-V2 and V4 hold, V3 is
  not required;
* device-detected errors are latched and returned by rcm_sync_status
  (validate = 1: bad CSR; validate = 2: asymmetric pattern; a tiny queue:
  capacity), and the plan stays usable afterwards."""
from __future__ import annotations

import numpy as np
import pytest

import mutate
import oracle
import synth
from verifier import verify

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

BAD_CSR, NOT_SYM, CAPACITY = 2, 3, 5


@pytest.fixture(scope="module")
def rcm():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_mlakarwps21_b200 as m
    return m


def _t(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _run(rcm, g, mode, start, **opts):
    plan = rcm.Plan(max(g.n, 1), max(g.nnz, 1), **opts)
    perm = plan.reorder(_t(g.row_ptr), _t(g.col_idx), mode, start).cpu().numpy()
    plan.close()
    return perm


PATHS = {
    "default": dict(),
    "chain": dict(flags=8, solo_threshold=-1),
    "serial": dict(flags=8 | 16, solo_threshold=-1),
    "multi": dict(flags=8 | 64, solo_threshold=-1),
    "leveled": dict(flags=8 | 32, solo_threshold=-1),
    "chain_small": dict(flags=8, solo_threshold=-1, batch_nodes=5, temp_elems=2304),
}


def _tiny():
    return [synth.grid2d(9, 7), synth.relabel(synth.grid3d_27(6, 5, 4), synth.randperm(120, 3)),
            synth.gnp(90, 0.06, 4), synth.star(40), synth.complete(12),
            synth.disjoint_union([synth.star(20), synth.path(6), synth.complete(5), synth.path(1)])]


@pytest.mark.parametrize("kind", list(mutate.ALL))
@pytest.mark.parametrize("path", list(PATHS))
def test_duplicates_loops_unsorted_tiny(rcm, kind, path):
    for i, g in enumerate(_tiny()):
        h = mutate.mutate(g, 100 + i, **mutate.ALL[kind])
        for mode, s in ((oracle.FIXED, h.n // 2), (oracle.MIN_DEGREE, 0), (oracle.PSEUDO_PERIPHERAL, 0)):
            ref = oracle.rcm(h.row_ptr, h.col_idx, mode, s)
            assert np.array_equal(_run(rcm, h, mode, s, **PATHS[path]), ref), (kind, path, i, mode)


@pytest.mark.parametrize("cfg", [2, 3, 4])
def test_duplicates_loops_unsorted_twins(rcm, cfg):
    g, mode, start = synth.config_graph(cfg, "small")
    h = mutate.mutate(g, 7 + cfg, **mutate.ALL["all"])
    ref = oracle.rcm(h.row_ptr, h.col_idx, mode, start)
    for path in ("default", "chain", "serial"):
        assert np.array_equal(_run(rcm, h, mode, start, **PATHS[path]), ref), path


def test_duplicates_loops_unsorted_batched(rcm):
    mats = [mutate.mutate(synth.c5_matrix(k, n), 300 + k, **mutate.ALL["all"])
            for k, n in enumerate([1000, 2500, 1200, 4000, 60, 9000])]
    b = synth.batch_of(mats)
    ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, oracle.MIN_DEGREE)
    total, nnz = int(b.node_off[-1]), int(b.nnz_off[-1])
    plan = rcm.Plan(total, nnz)
    perm = plan.reorder_batched(_t(b.node_off), _t(b.nnz_off), _t(b.row_ptr_local), _t(b.col_idx_local),
                                total, nnz).cpu().numpy()
    plan.close()
    assert np.array_equal(perm, ref)


@pytest.mark.parametrize("path", ["default", "leveled"])
@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
def test_pseudo_peripheral_full_configs(rcm, cfg, path):
    g, mode, start = synth.config_graph(cfg)
    ref = oracle.rcm(g.row_ptr, g.col_idx, oracle.PSEUDO_PERIPHERAL, 0)
    got = _run(rcm, g, oracle.PSEUDO_PERIPHERAL, 0, **PATHS[path])
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
def test_find_pseudo_peripheral_full_size(rcm, cfg):
    """rcm_find_pseudo_peripheral from the MIN_DEGREE seed of the largest
    component and from node 0, against oracle.gl (C-5)."""
    g, _, _ = synth.config_graph(cfg)
    deg = np.diff(g.row_ptr)
    big = int(np.argmax(deg))          # a node of the giant component
    plan = rcm.Plan(g.n, g.nnz)
    rp, ci = _t(g.row_ptr), _t(g.col_idx)
    for r in (0, big):
        assert plan.find_pseudo_peripheral(rp, ci, r) == oracle.gl(g.row_ptr, g.col_idx, r), r
    plan.close()


@pytest.mark.parametrize("path", ["default", "chain", "serial", "multi"])
def test_no_sort_emits_a_bfs_order(rcm, path):
    for cfg in (1, 2, 4):
        g, mode, start = synth.config_graph(cfg, "small")
        opts = dict(PATHS[path])
        opts["flags"] = opts.get("flags", 0) | 4
        perm = _run(rcm, g, mode, start, **opts)
        assert verify(g.row_ptr, g.col_idx, perm, mode, start, check_sort=False) is None, (cfg, path)


def _status(rcm, plan, g, mode=oracle.MIN_DEGREE, start=0, nnz=None):
    perm = torch.empty(g.n, dtype=torch.int32, device="cuda")
    rcm.rcm_reorder(plan.handle, g.n, g.nnz if nnz is None else nnz, _t(g.row_ptr), _t(g.col_idx), mode,
                    start, perm)
    return rcm.rcm_sync_status(plan.handle), perm


def _recover(rcm, plan, g):
    st, perm = _status(rcm, plan, g)
    assert st == 0
    assert np.array_equal(perm.cpu().numpy(), oracle.rcm(g.row_ptr, g.col_idx, oracle.MIN_DEGREE))


@pytest.mark.parametrize("path", ["default", "chain"])
def test_validate_bad_csr_is_latched(rcm, path):
    g = synth.relabel(synth.grid2d(30, 20), synth.randperm(600, 5))
    plan = rcm.Plan(g.n, g.nnz + 16, validate=1, **PATHS[path])
    bad = synth.CSR(g.n, g.row_ptr.copy(), g.col_idx.copy())
    bad.row_ptr[100] = bad.row_ptr[101] + 1             # non-monotone row_ptr
    assert _status(rcm, plan, bad)[0] == BAD_CSR
    _recover(rcm, plan, g)
    bad = synth.CSR(g.n, g.row_ptr.copy(), g.col_idx.copy())
    bad.col_idx[37] = g.n + 3                           # column out of range
    assert _status(rcm, plan, bad)[0] == BAD_CSR
    _recover(rcm, plan, g)
    assert _status(rcm, plan, g, nnz=g.nnz + 4)[0] == BAD_CSR   # row_ptr[n] != nnz
    _recover(rcm, plan, g)
    plan.close()


@pytest.mark.parametrize("path", ["default", "chain"])
def test_validate_asymmetric_is_latched(rcm, path):
    g = synth.relabel(synth.grid2d(30, 20), synth.randperm(600, 6))
    rows = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    drop = int(np.nonzero(rows != g.col_idx)[0][50])    # remove (u, c), keep (c, u)
    keep = np.ones(g.nnz, bool)
    keep[drop] = False
    rp = np.zeros(g.n + 1, np.int64)
    np.cumsum(np.bincount(rows[keep], minlength=g.n), out=rp[1:])
    asym = synth.CSR(g.n, rp.astype(np.int32), g.col_idx[keep].copy())
    plan = rcm.Plan(g.n, g.nnz, validate=2, **PATHS[path])
    assert _status(rcm, plan, asym)[0] == NOT_SYM
    _recover(rcm, plan, g)
    plan.close()
    plan = rcm.Plan(g.n, g.nnz, validate=1, **PATHS[path])   # validate = 1 does not check symmetry
    assert _status(rcm, plan, asym)[0] != NOT_SYM
    plan.close()


def test_queue_capacity_is_latched(rcm):
    g = synth.relabel(synth.grid3d_27(12, 12, 12), synth.randperm(1728, 8))
    plan = rcm.Plan(g.n, g.nnz, queue_capacity=4, flags=8, solo_threshold=-1)
    assert _status(rcm, plan, g)[0] == CAPACITY
    plan.close()


def test_batched_validate(rcm):
    """the batched path validates too (row_ptr, column range, starts)."""
    mats = [synth.c5_matrix(k, n) for k, n in enumerate([1000, 1500, 800])]
    b = synth.batch_of(mats)
    total, nnz = int(b.node_off[-1]), int(b.nnz_off[-1])
    plan = rcm.Plan(total, nnz, validate=1)
    args = lambda rp, ci: (_t(b.node_off), _t(b.nnz_off), _t(rp), _t(ci), total, nnz)  # noqa: E731
    perm = torch.empty(total, dtype=torch.int32, device="cuda")

    def st(rp, ci, mode=oracle.MIN_DEGREE, starts=None):
        rcm.rcm_reorder_batched(plan.handle, 3, total, nnz, *args(rp, ci)[:4], mode,
                                None if starts is None else _t(starts), perm)
        return rcm.rcm_sync_status(plan.handle)

    ci = b.col_idx_local.copy()
    ci[int(b.nnz_off[1]) + 5] = 1500 + 7                # out of matrix 1's range
    assert st(b.row_ptr_local, ci) == BAD_CSR
    assert st(b.row_ptr_local, b.col_idx_local) == 0
    starts = np.array([0, 1500, 3], np.int32)           # start of matrix 1 out of range
    assert st(b.row_ptr_local, b.col_idx_local, oracle.FIXED, starts) == BAD_CSR
    rp = b.row_ptr_local.copy()
    rp[1000 + 1 + 40] = rp[1000 + 1 + 41] + 2           # non-monotone row_ptr in matrix 1
    assert st(rp, b.col_idx_local) == BAD_CSR
    assert st(b.row_ptr_local, b.col_idx_local) == 0
    ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, oracle.MIN_DEGREE)
    assert np.array_equal(perm.cpu().numpy(), ref)
    plan.close()


def test_batched_single_node_and_disconnected_matrices(rcm):
    """a batch that is mostly 1-node matrices, and a matrix with
    many components (a 50,000-node diagonal) next to ordinary meshes."""
    diag = synth.CSR(50000, np.arange(50001, dtype=np.int32), np.arange(50000, dtype=np.int32))
    mats = [synth.path(1)] * 300 + [synth.c5_matrix(3, 2000), diag, synth.path(2), synth.path(1)]
    mats += [synth.disjoint_union([synth.path(3), synth.path(1), synth.star(4)] * 50)]
    b = synth.batch_of(mats)
    total, nnz = int(b.node_off[-1]), int(b.nnz_off[-1])
    for mode in (oracle.MIN_DEGREE, oracle.PSEUDO_PERIPHERAL):
        ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, mode)
        plan = rcm.Plan(total, nnz)
        perm = plan.reorder_batched(_t(b.node_off), _t(b.nnz_off), _t(b.row_ptr_local), _t(b.col_idx_local),
                                    total, nnz, mode=mode).cpu().numpy()
        plan.close()
        assert np.array_equal(perm, ref), mode


def test_hub_above_the_claims_bitmap(rcm):
    """a row longer than the shared-memory claims bitmap (64 (T+1)
    entries) must not fail with RCM_ERR_CAPACITY (the paper's histogram method
    has no valence limit)."""
    g = synth.relabel(synth.star(700000), synth.randperm(700001, 9))
    ref = oracle.rcm(g.row_ptr, g.col_idx, oracle.MIN_DEGREE)
    for path in ("default", "chain", "serial", "leveled"):
        assert np.array_equal(_run(rcm, g, oracle.MIN_DEGREE, 0, **PATHS[path]), ref), path


def test_leveled_wide_levels_and_overflow(rcm):
    """Leveled schedule (NEXT-3) under stress: a level of 5,920 parents of
    valence ~1,200 > T/2 (one batch each: 40 batches per block and round, so
    the block's output list is merged), rounds (level wider than blocks x B_s),
    a skewed output (every grandchild written by few blocks is re-spread), per
    block outputs above the shared-memory buffer (HBM scratch), long rows in the
    block-wide discovery pass, duplicate entries (test-side mutator)."""
    rng = np.random.default_rng(21)
    P, deg, G = 5920, 1200, 400_000
    par = np.repeat(np.arange(1, P + 1), deg)
    gc = 1 + P + rng.integers(0, G, P * deg)
    src = np.concatenate([np.zeros(P, np.int64), par])
    dst = np.concatenate([np.arange(1, P + 1), gc])
    g = synth.csr_from_pairs(1 + P + G, src, dst)
    g = mutate.mutate(g, 22, dup=0.01)
    ref = oracle.rcm(g.row_ptr, g.col_idx, oracle.FIXED, 0)
    opts = dict(flags=8 | 32, solo_threshold=-1, blocks_per_sm=1, temp_elems=2304, batch_nodes=64)
    assert np.array_equal(_run(rcm, g, oracle.FIXED, 0, **opts), ref)
    assert np.array_equal(_run(rcm, g, oracle.FIXED, 0, **PATHS["leveled"]), ref)


def test_batched_matrices_above_the_shared_bitmap(rcm):
    """Matrices above 2^17 - 1 nodes keep their visited bitmaps in HBM, packed
    over all nodes (neighbouring matrices share boundary words); with an
    oversize hub and PSEUDO_PERIPHERAL."""
    mats = [synth.relabel(synth.grid2d(400, 350), synth.randperm(140000, 11)), synth.path(37),
            synth.relabel(synth.star(140000), synth.randperm(140001, 12)), synth.c5_matrix(5, 3000),
            synth.relabel(synth.grid3d_27(53, 50, 50), synth.randperm(132500, 13))]
    b = synth.batch_of(mats)
    total, nnz = int(b.node_off[-1]), int(b.nnz_off[-1])
    for mode in (oracle.MIN_DEGREE, oracle.PSEUDO_PERIPHERAL):
        ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, mode, threads=4)
        plan = rcm.Plan(total, nnz, flags=rcm.RCM_FLAG_BATCHED_ONLY)
        perm = plan.reorder_batched(_t(b.node_off), _t(b.nnz_off), _t(b.row_ptr_local), _t(b.col_idx_local),
                                    total, nnz, mode=mode).cpu().numpy()
        plan.close()
        for k in range(len(mats)):
            a0, a1 = int(b.node_off[k]), int(b.node_off[k + 1])
            assert np.array_equal(perm[a0:a1], ref[a0:a1]), (mode, k)


def test_small_graph_with_a_large_csr(rcm):
    """rcm_reorder on a graph of <= solo_threshold nodes whose CSR does not fit
    in shared memory takes the global-memory one-block path (k_solo) instead
    of the staged one (k_solo_sm); both must give the oracle's order."""
    for g in (synth.complete(900), synth.gnp(3000, 0.05, 17, diag=True),
              mutate.mutate(synth.gnp(2000, 0.08, 18), 19, **mutate.ALL["all"])):
        assert 4 * (g.n + 1 + g.nnz) > 200 * 1024
        for mode, s in ((oracle.FIXED, g.n // 3), (oracle.MIN_DEGREE, 0), (oracle.PSEUDO_PERIPHERAL, 0)):
            ref = oracle.rcm(g.row_ptr, g.col_idx, mode, s)
            assert np.array_equal(_run(rcm, g, mode, s), ref), (g.n, mode)


@pytest.mark.parametrize("chunks", [1, 3, 8])
def test_batched_host_pipeline(rcm, chunks):
    """rcm_reorder_batched_host: host batch in, host permutations out, copies
    overlapped with the ordering in `chunks` ranges; same result as the oracle
    (and as the device API) for MIN_DEGREE, FIXED and PSEUDO_PERIPHERAL."""
    mats = [synth.c5_matrix(k, n) for k, n in enumerate([1000, 2600, 1200, 4100, 900, 7000, 1500, 3300, 2000])]
    mats.append(mutate.mutate(synth.c5_matrix(9, 1800), 5, **mutate.ALL["all"]))
    b = synth.batch_of(mats)
    num, total, nnz = len(mats), int(b.node_off[-1]), int(b.nnz_off[-1])
    h = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
    starts = ((np.arange(num) * 7919) % np.diff(b.node_off)).astype(np.int32)
    plan = rcm.Plan(total, nnz, flags=rcm.RCM_FLAG_BATCHED_ONLY)
    for mode in (oracle.MIN_DEGREE, oracle.FIXED, oracle.PSEUDO_PERIPHERAL):
        ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, mode,
                                 starts if mode == oracle.FIXED else None)
        perm_h = torch.empty(total, dtype=torch.int32).pin_memory()
        dev = dict(node_off_d=torch.empty(num + 1, dtype=torch.int64, device="cuda"),
                   nnz_off_d=torch.empty(num + 1, dtype=torch.int64, device="cuda"),
                   row_ptr_d=torch.empty(b.row_ptr_local.size, dtype=torch.int32, device="cuda"),
                   col_idx_d=torch.empty(nnz, dtype=torch.int32, device="cuda"),
                   starts_d=torch.empty(num, dtype=torch.int32, device="cuda") if mode == oracle.FIXED else None,
                   perm_d=torch.empty(total, dtype=torch.int32, device="cuda"))
        rcm.rcm_reorder_batched_host(plan.handle, num, h(b.node_off), h(b.nnz_off), h(b.row_ptr_local),
                                     h(b.col_idx_local), mode, h(starts) if mode == oracle.FIXED else None, perm_h,
                                     chunks=chunks, **dev)
        assert rcm.rcm_sync_status(plan.handle) == 0
        assert np.array_equal(perm_h.numpy(), ref), (mode, chunks)
    plan.close()


@pytest.mark.parametrize("path", ["default", "chain", "leveled"])
def test_isolated_nodes(rcm, path):
    """Isolated nodes (valence 0) take the first component positions in id
    order directly (components phase fast path, C-6): an edgeless graph, and
    isolated nodes interleaved with grids, stars and paths under a relabelling,
    for FIXED (a non-isolated start), MIN_DEGREE and PSEUDO_PERIPHERAL."""
    empty = synth.csr_from_pairs(1000, np.zeros(0, np.int64), np.zeros(0, np.int64))
    parts = [synth.grid2d(15, 9), synth.path(1), synth.star(25), synth.path(1), synth.path(1),
             synth.relabel(synth.grid3d_27(5, 5, 4), synth.randperm(100, 7)), synth.path(1), synth.path(9)]
    mixed = synth.relabel(synth.disjoint_union(parts), synth.randperm(sum(p.n for p in parts), 8))
    for g in (empty, mixed):
        starts = [(oracle.MIN_DEGREE, 0), (oracle.PSEUDO_PERIPHERAL, 0)]
        if g.nnz:
            starts.append((oracle.FIXED, int(np.argmax(np.diff(g.row_ptr)))))
        for mode, s0 in starts:
            ref = oracle.rcm(g.row_ptr, g.col_idx, mode, s0)
            assert np.array_equal(_run(rcm, g, mode, s0, **PATHS[path]), ref), (g.n, mode)
