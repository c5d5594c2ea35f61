"""Tiny inputs through every path, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): look-back chain, serial chain, multi-batch, leveled,
the one-block solo path, batched (incl. an oversize parent and PSEUDO_PERIPHERAL),
components.  Each result is checked against the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm

t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
g = synth.relabel(synth.grid3d_27(9, 8, 7), synth.randperm(504, 3))
mix = synth.relabel(synth.disjoint_union([synth.grid2d(12, 9), synth.star(40), synth.path(1), synth.complete(6)]),
                    synth.randperm(108 + 41 + 1 + 6, 4))
bad = 0
for name, opts in [("lookback", dict(flags=8, solo_threshold=-1, blocks_per_sm=1)),
                   ("serial", dict(flags=8 | 16, solo_threshold=-1, blocks_per_sm=1)),
                   ("multi", dict(flags=8 | 64, solo_threshold=-1, blocks_per_sm=1)),
                   ("leveled", dict(flags=8 | 32, solo_threshold=-1, blocks_per_sm=1)),
                   ("solo", dict())]:
    for gg, mode in ((g, oracle.MIN_DEGREE), (mix, oracle.MIN_DEGREE), (mix, oracle.PSEUDO_PERIPHERAL)):
        plan = rcm.Plan(gg.n, gg.nnz, **opts)
        got = plan.reorder(t(gg.row_ptr), t(gg.col_idx), mode, 0).cpu().numpy()
        plan.close()
        ok = np.array_equal(got, oracle.rcm(gg.row_ptr, gg.col_idx, mode, 0))
        bad += not ok
        print(name, gg.n, mode, "ok" if ok else "MISMATCH", flush=True)
b = synth.batch_of([synth.c5_matrix(k, n) for k, n in enumerate([300, 1200, 700])] + [synth.star(1500), mix])
total, nnz = int(b.node_off[-1]), int(b.nnz_off[-1])
for mode in (oracle.MIN_DEGREE, oracle.PSEUDO_PERIPHERAL):
    plan = rcm.Plan(total, nnz, flags=rcm.RCM_FLAG_BATCHED_ONLY)
    got = plan.reorder_batched(t(b.node_off), t(b.nnz_off), t(b.row_ptr_local), t(b.col_idx_local), total, nnz,
                               mode=mode).cpu().numpy()
    plan.close()
    ok = np.array_equal(got, oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, mode))
    bad += not ok
    print("batched", total, mode, "ok" if ok else "MISMATCH", flush=True)
print("ALL OK" if bad == 0 else f"{bad} MISMATCHES")
