"""CPU: the ABI's edge-case inputs (duplicates, self-loops, unsorted rows; built
by tests/mutate.py) against the oracle's pins.  Column order inside a row must
not change the result (C-1: children are sorted by (valence, id));
duplicates and self-loops count in the valence (C-2) and are skipped as
children (C-8), so the oracle's order on a mutated graph must pass
the independent verifier V0-V4 computed with the mutated valences."""
import numpy as np
import pytest

import mutate
import oracle
import synth
from verifier import verify


def _graphs():
    return [synth.grid2d(9, 7), synth.relabel(synth.grid3d_27(6, 5, 4), synth.randperm(120, 3)),
            synth.gnp(90, 0.06, 4), synth.disjoint_union([synth.star(20), synth.path(6), synth.complete(5)]),
            synth.config_graph(4, "small")[0]]


@pytest.mark.parametrize("mode", [oracle.FIXED, oracle.MIN_DEGREE, oracle.PSEUDO_PERIPHERAL])
def test_shuffled_rows_do_not_change_the_order(mode):
    for i, g in enumerate(_graphs()):
        h = mutate.unsorted(g, 10 + i)
        assert not all(np.all(np.diff(h.col_idx[h.row_ptr[v]:h.row_ptr[v + 1]]) > 0) for v in range(h.n))
        s = g.n // 3
        assert np.array_equal(oracle.rcm(h.row_ptr, h.col_idx, mode, s), oracle.rcm(g.row_ptr, g.col_idx, mode, s))


@pytest.mark.parametrize("kind", ["dup", "loops", "all"])
@pytest.mark.parametrize("mode", [oracle.FIXED, oracle.MIN_DEGREE, oracle.PSEUDO_PERIPHERAL])
def test_duplicates_and_loops_pass_the_verifier(kind, mode):
    for i, g in enumerate(_graphs()):
        h = mutate.mutate(g, 20 + i, **mutate.ALL[kind])
        assert h.nnz > g.nnz
        # valences are the raw row lengths of the mutated CSR (C-2)
        assert np.array_equal(oracle.degree(h.row_ptr), np.diff(h.row_ptr))
        perm = oracle.rcm(h.row_ptr, h.col_idx, mode, g.n // 2)
        assert verify(h.row_ptr, h.col_idx, perm, mode, g.n // 2) is None
