"""CPU-only: the host CPU-BATCH (include/rcm_cpu.h) --
Alg. 5 on std::thread workers -- returns exactly the oracle's serial RCM
permutation, for every thread count and batch limit (C-11), on the
tiny families, the small config twins, disconnected graphs and all start modes."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def cb():
    import importlib.util
    spec = importlib.util.spec_from_file_location("_b", os.path.join(ROOT, "paper_conf_ipps_mlakarwps21_b200", "build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    b.build_cpu()
    from paper_conf_ipps_mlakarwps21_b200 import cpu_batch
    return cpu_batch


def _tiny():
    gs = [synth.path(1), synth.path(2), synth.path(7), synth.cycle(9), synth.star(12), synth.complete(9),
          synth.binary_tree(63), synth.grid2d(7, 5), synth.grid2d(13, 40, True)]
    gs += [synth.gnp(80, 0.05, s) for s in range(6)]
    gs += [synth.gnp(60, 0.3, 50 + s, diag=True) for s in range(2)]
    gs.append(synth.relabel(synth.grid3d_27(7, 6, 5), synth.randperm(210, 3)))
    gs.append(synth.disjoint_union([synth.path(4), synth.star(30), synth.complete(5), synth.path(1),
                                    synth.grid2d(9, 9)]))
    return gs


def test_header_symbols_exported(cb):
    src = re.sub(r"/\*.*?\*/", "", open(os.path.join(ROOT, "include", "rcm_cpu.h")).read(), flags=re.S)
    names = sorted(set(re.findall(r"\b(rcm_[a-z_]+)\s*\(", src)))
    assert names == ["rcm_cpu_batch"]
    out = subprocess.run(["nm", "-D", "--defined-only", cb.LIB_PATH], capture_output=True, text=True).stdout
    for name in names:
        assert re.search(rf"\bT {name}$", out, flags=re.M), name


@pytest.mark.parametrize("threads,bn,te", [(1, 0, 0), (3, 1, 16), (8, 3, 64), (8, 0, 0)])
def test_tiny_families(cb, threads, bn, te):
    for g in _tiny():
        for mode, start in ((oracle.FIXED, g.n // 2), (oracle.MIN_DEGREE, 0), (oracle.PSEUDO_PERIPHERAL, 0)):
            ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
            perm = cb.rcm_cpu_batch(g.row_ptr, g.col_idx, mode, start, threads=threads, batch_nodes=bn, temp_elems=te)
            assert np.array_equal(perm, ref), (g.n, mode, threads, bn)


@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
def test_config_small_twins(cb, cfg):
    g, mode, start = synth.config_graph(cfg, "small")
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    for threads in (2, 8):
        for bn in (0, 5):
            perm, st = cb.rcm_cpu_batch(g.row_ptr, g.col_idx, mode, start, threads=threads, batch_nodes=bn,
                                        with_stats=True)
            assert np.array_equal(perm, ref), (cfg, threads, bn)
            # every executed batch rediscovered either early or late (Alg. 5 ln 5-19)
            assert st["rediscover_early"] + st["rediscover_late"] == st["batches_executed"]


def test_full_c2_parity(cb):
    g, mode, start = synth.config_graph(2)
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    perm, st = cb.rcm_cpu_batch(g.row_ptr, g.col_idx, mode, start, threads=8, with_stats=True)
    assert np.array_equal(perm, ref)
    assert st["chains"] == 1


def test_argument_errors(cb):
    g = synth.path(5)
    with pytest.raises(RuntimeError):
        cb.rcm_cpu_batch(g.row_ptr, g.col_idx, oracle.FIXED, 7)
    with pytest.raises(RuntimeError):
        cb.rcm_cpu_batch(g.row_ptr, g.col_idx, 3, 0)
