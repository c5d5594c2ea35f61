"""GPU parity: the CUDA path (through the C ABI) vs the serial oracle, element by
element (bit-exact: the output is an integer permutation).  Run with -m gpu."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from verifier import verify

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def rcm():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_mlakarwps21_b200 as m
    return m


def _dev(g):
    return (torch.from_numpy(np.ascontiguousarray(g.row_ptr)).cuda(),
            torch.from_numpy(np.ascontiguousarray(g.col_idx)).cuda())


def _run(rcm, g, mode, start, plan=None, **opts):
    own = plan is None
    if own:
        plan = rcm.Plan(max(g.n, 1), max(g.nnz, 1), **opts)
    rp, ci = _dev(g)
    iperm = torch.empty(g.n, dtype=torch.int32, device="cuda")
    perm = plan.reorder(rp, ci, mode, start, iperm=iperm).cpu().numpy()
    ip = iperm.cpu().numpy()
    assert np.array_equal(ip[perm], np.arange(g.n))
    stats = plan.stats()
    if own:
        plan.close()
    return perm, stats


def _tiny_graphs():
    gs = [synth.path(1), synth.path(2), synth.path(7), synth.cycle(9), synth.star(12), synth.complete(9),
          synth.binary_tree(63), synth.grid2d(7, 5), synth.grid2d(13, 40, True)]
    gs += [synth.gnp(80, 0.05, s) for s in range(6)]
    gs += [synth.gnp(60, 0.3, 50 + s, diag=True) for s in range(2)]
    gs.append(synth.relabel(synth.grid3d_27(7, 6, 5), synth.randperm(210, 3)))
    gs.append(synth.disjoint_union([synth.path(4), synth.star(30), synth.complete(5), synth.path(1),
                                    synth.grid2d(9, 9)]))
    return gs


MODES = [(oracle.FIXED, "mid"), (oracle.MIN_DEGREE, None)]
PATHS = {
    "solo": dict(),
    "chain": dict(flags=8, solo_threshold=-1),                       # look-back chain (default)
    "chain_bs1": dict(flags=8, solo_threshold=-1, batch_nodes=1),
    "chain_noearly": dict(flags=8 | 2, solo_threshold=-1, batch_nodes=7, temp_elems=2304),
    "serial": dict(flags=8 | 16, solo_threshold=-1),                 # Alg. 5 hand-off chain
    "serial_bs3_noovh": dict(flags=8 | 16 | 1, solo_threshold=-1, batch_nodes=3),
    "serial_noearly": dict(flags=8 | 16 | 2, solo_threshold=-1, batch_nodes=7, temp_elems=2304),
    "leveled": dict(flags=8 | 32, solo_threshold=-1),                # Alg. 2 (NEXT-3)
    "multi": dict(flags=8 | 64, solo_threshold=-1),                  # multi-batch execution (NEXT-2)
    "multi_bs3_noearly": dict(flags=8 | 64 | 2, solo_threshold=-1, batch_nodes=3, temp_elems=2304),
}


@pytest.mark.parametrize("path", list(PATHS))
def test_tiny_families(rcm, path):
    for g in _tiny_graphs():
        for mode, s in MODES:
            start = g.n // 2 if s == "mid" else 0
            ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
            got, _ = _run(rcm, g, mode, start, **PATHS[path])
            assert np.array_equal(got, ref), (path, g.n, mode)


@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
@pytest.mark.parametrize("path", ["solo", "chain", "serial", "serial_bs3_noovh", "leveled"])
def test_config_small_twins(rcm, cfg, path):
    g, mode, start = synth.config_graph(cfg, "small")
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    opts = dict(PATHS[path])
    if path == "solo":
        opts["solo_threshold"] = g.n
    got, st = _run(rcm, g, mode, start, **opts, collect_stats=1)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("opts", [
    dict(batch_nodes=1), dict(batch_nodes=2), dict(batch_nodes=3), dict(batch_nodes=64),
    dict(batch_nodes=1024), dict(temp_elems=2304), dict(blocks_per_sm=1), dict(flags=1), dict(flags=2),
    dict(flags=3, batch_nodes=16, temp_elems=2304), dict(flags=16), dict(flags=16, batch_nodes=1),
    dict(flags=16 | 1), dict(flags=16 | 2), dict(flags=16, blocks_per_sm=1, batch_nodes=1024),
])
def test_sweep_invariance(rcm, opts):
    g, mode, start = synth.config_graph(2, "small")
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    o = dict(solo_threshold=-1)
    o.update(opts)
    got, _ = _run(rcm, g, mode, start, **o)
    assert np.array_equal(got, ref), opts


def test_repeat_determinism_and_stats(rcm):
    g, mode, start = synth.config_graph(2, "small")
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    plan = rcm.Plan(g.n, g.nnz, solo_threshold=-1, collect_stats=1, batch_nodes=64)
    plan2 = rcm.Plan(g.n, g.nnz, solo_threshold=-1, collect_stats=1, batch_nodes=64, flags=16)
    rp, ci = _dev(g)
    for it in range(40):
        plan, plan2 = plan2, plan
        perm = plan.reorder(rp, ci, mode, start).cpu().numpy()
        assert np.array_equal(perm, ref)
        st = plan.stats()
        # Fig. 3 semantics: generated >= dequeued >= executed
        assert st["batches_generated"] + 1 >= st["batches_dequeued"] >= st["batches_executed"]
        assert st["batches_executed"] + st["batches_empty"] <= st["batches_dequeued"]
        assert st["components"] == 1
    plan.close()
    plan2.close()


@pytest.mark.parametrize("cfg", [1, 2])
def test_full_config_parity(rcm, cfg):
    g, mode, start = synth.config_graph(cfg)
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    got, st = _run(rcm, g, mode, start, collect_stats=1)
    assert np.array_equal(got, ref)
    assert verify(g.row_ptr, g.col_idx, got, mode, start) is None


@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
def test_full_config_parity_leveled(rcm, cfg):
    """NEXT-3: Alg. 2 on the GPU -- a second, independent implementation."""
    g, mode, start = synth.config_graph(cfg)
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    got, _ = _run(rcm, g, mode, start, flags=8 | 32, solo_threshold=-1)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
def test_full_config_parity_multi_batch(rcm, cfg):
    """NEXT-2: two batches in flight per block -- result-neutral (C-11)."""
    g, mode, start = synth.config_graph(cfg)
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    got, _ = _run(rcm, g, mode, start, flags=8 | 64, solo_threshold=-1)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("cfg", [3, 4])
def test_full_config_parity_disconnected(rcm, cfg):
    g, mode, start = synth.config_graph(cfg)
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    got, st = _run(rcm, g, mode, start, collect_stats=1)
    assert np.array_equal(got, ref)


def test_gl_finder(rcm):
    for g, r in [(synth.path(30), 0), (synth.grid2d(7, 5), 0), (synth.grid2d(40, 13), 0)]:
        plan = rcm.Plan(g.n, g.nnz)
        rp, ci = _dev(g)
        assert plan.find_pseudo_peripheral(rp, ci, r) == oracle.gl(g.row_ptr, g.col_idx, r)
        plan.close()
    g, _, _ = synth.config_graph(2, "small")
    plan = rcm.Plan(g.n, g.nnz, solo_threshold=-1)
    rp, ci = _dev(g)
    for r in [0, 17, 4000]:
        assert plan.find_pseudo_peripheral(rp, ci, r) == oracle.gl(g.row_ptr, g.col_idx, r)
    perm = plan.reorder(rp, ci, oracle.PSEUDO_PERIPHERAL, 0).cpu().numpy()
    assert np.array_equal(perm, oracle.rcm(g.row_ptr, g.col_idx, oracle.PSEUDO_PERIPHERAL, 0))
    plan.close()


def test_batched_small(rcm):
    b = synth.c5_batch(num=40, seed=5, lo=50, hi=3000)
    ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, oracle.MIN_DEGREE)
    total, nnz = int(b.node_off[-1]), int(b.nnz_off[-1])
    plan = rcm.Plan(total, nnz)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
    perm = plan.reorder_batched(t(b.node_off), t(b.nnz_off), t(b.row_ptr_local), t(b.col_idx_local),
                                total, nnz).cpu().numpy()
    assert np.array_equal(perm, ref)
    # FIXED starts
    starts = (np.arange(40) * 7919) % np.diff(b.node_off)
    ref2 = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, oracle.FIXED, starts)
    perm2 = plan.reorder_batched(t(b.node_off), t(b.nnz_off), t(b.row_ptr_local), t(b.col_idx_local),
                                 total, nnz, mode=oracle.FIXED, starts=t(starts.astype(np.int32))).cpu().numpy()
    assert np.array_equal(perm2, ref2)
    plan.close()


def test_host_argument_errors(rcm):
    g = synth.path(5)
    plan = rcm.Plan(5, 8)
    rp, ci = _dev(g)
    perm = torch.empty(5, dtype=torch.int32, device="cuda")
    with pytest.raises(rcm.RCMError):
        rcm.rcm_reorder(plan.handle, 5, 8, rp, ci, oracle.FIXED, 7, perm)      # start out of range
    with pytest.raises(rcm.RCMError):
        rcm.rcm_reorder(plan.handle, 6, 8, rp, ci, oracle.FIXED, 0, perm)      # n above plan
    plan.close()


@pytest.mark.parametrize("opts", [dict(), dict(batch_nodes=64), dict(flags=16), dict(flags=64)])
def test_stress_no_stall_and_determinism(rcm, opts):
    """Repeated runs on one plan: early termination races (a worker abandoning an
    unpublished slot while others are mid look-back) must never stall; every
    run must be bit-identical."""
    import time
    g, mode, start = synth.config_graph(2, "small")
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    plan = rcm.Plan(g.n, g.nnz, solo_threshold=-1, **opts)
    rp, ci = _dev(g)
    perm = torch.empty(g.n, dtype=torch.int32, device="cuda")
    t0 = time.time()
    for _ in range(300):
        rcm.rcm_reorder(plan.handle, g.n, g.nnz, rp, ci, mode, start, perm)
    assert rcm.rcm_sync_status(plan.handle) == 0
    assert time.time() - t0 < 60
    assert np.array_equal(perm.cpu().numpy(), ref)
    for _ in range(20):
        plan.reorder(rp, ci, mode, start, perm=perm)
        assert np.array_equal(perm.cpu().numpy(), ref)
    plan.close()


def test_c5_device_generator_matches_numpy(rcm):
    import synth.device as sd
    mats = [0, 1, 2, 3, 17, 4000]
    b = sd.c5_generate(mats, num=8192)
    sizes = synth.c5_sizes(8192)
    rp = b["row_ptr_local"].cpu().numpy()
    ci = b["col_idx_local"].cpu().numpy()
    for i, k in enumerate(mats):
        g = synth.c5_matrix(k, int(sizes[k]))
        a, e = int(b["node_off_h"][i]), int(b["node_off_h"][i + 1])
        assert np.array_equal(rp[a + i: e + i + 1], g.row_ptr)
        assert np.array_equal(ci[int(b["nnz_off_h"][i]): int(b["nnz_off_h"][i + 1])], g.col_idx)
    # and the batched traversal of the device-generated matrices
    plan = rcm.Plan(b["total"], b["total_nnz"])
    perm = plan.reorder_batched(b["node_off"], b["nnz_off"], b["row_ptr_local"], b["col_idx_local"],
                                b["total"], b["total_nnz"]).cpu().numpy()
    for i, k in enumerate(mats):
        g = synth.c5_matrix(k, int(sizes[k]))
        a, e = int(b["node_off_h"][i]), int(b["node_off_h"][i + 1])
        assert np.array_equal(perm[a:e], oracle.rcm(g.row_ptr, g.col_idx, oracle.MIN_DEGREE))
    plan.close()


def test_batched_pseudo_peripheral(rcm):
    b = synth.c5_batch(num=12, seed=7, lo=30, hi=900)
    ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, oracle.PSEUDO_PERIPHERAL)
    total, nnz = int(b.node_off[-1]), int(b.nnz_off[-1])
    plan = rcm.Plan(total, nnz)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
    perm = plan.reorder_batched(t(b.node_off), t(b.nnz_off), t(b.row_ptr_local), t(b.col_idx_local),
                                total, nnz, mode=oracle.PSEUDO_PERIPHERAL).cpu().numpy()
    assert np.array_equal(perm, ref)
    plan.close()


def test_disconnected_pseudo_peripheral(rcm):
    g = synth.disjoint_union([synth.grid2d(9, 7), synth.path(12), synth.star(5), synth.path(1),
                              synth.relabel(synth.grid3d_27(5, 4, 6), synth.randperm(120, 3))])
    g = synth.relabel(g, synth.randperm(g.n, 21))
    ref = oracle.rcm(g.row_ptr, g.col_idx, oracle.PSEUDO_PERIPHERAL, 0)
    for opts in [dict(), dict(solo_threshold=-1, flags=8), dict(solo_threshold=8, flags=8)]:
        got, _ = _run(rcm, g, oracle.PSEUDO_PERIPHERAL, 0, **opts)
        assert np.array_equal(got, ref), opts


def _cc_mixes():
    """Disconnected graphs for the components phase (a13): a dominant component
    the sampled union-find skips (a relabelled grid, or a hub star whose row
    exceeds the block-per-row threshold) next to hubs, cliques, paths and
    isolated nodes, ids shuffled so members and non-members interleave."""
    small = [synth.path(1), synth.path(2), synth.path(5), synth.complete(40), synth.star(100),
             synth.cycle(33), synth.path(1), synth.binary_tree(31)]
    mixes = [synth.disjoint_union([synth.grid3d_27(20, 20, 20, diag=False), synth.star(5000)] + small),
             synth.disjoint_union([synth.star(20000), synth.grid2d(30, 30)] + small * 3),
             synth.disjoint_union(small * 40)]
    return [synth.relabel(g, synth.randperm(g.n, 70 + i)) for i, g in enumerate(mixes)]


@pytest.mark.parametrize("path", ["chain", "serial", "multi", "leveled"])
def test_components_sampled_union_find(rcm, path):
    for g in _cc_mixes():
        for mode, start in ((oracle.MIN_DEGREE, 0), (oracle.FIXED, g.n // 3), (oracle.PSEUDO_PERIPHERAL, 0)):
            ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
            got, st = _run(rcm, g, mode, start, collect_stats=1, **PATHS[path])
            assert np.array_equal(got, ref), (path, g.n, mode)
