"""Localise a solo-path mismatch: run small graphs through the one-block path
and report the first differing position against the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm

def run(g, mode, start, **o):
    plan = rcm.Plan(g.n, max(g.nnz, 1), solo_threshold=g.n, **o)
    p = plan.reorder(torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda(), mode, start).cpu().numpy()
    plan.close()
    return p

cases = {"c4twin": synth.config_graph(4, "small"), "c3twin": synth.config_graph(3, "small"),
         "star3000": (synth.star(3000), 1, 0), "star1500+path": (synth.disjoint_union([synth.star(1500), synth.path(9)]), 1, 0),
         "star1000": (synth.star(1000), 1, 0), "star1030": (synth.star(1030), 1, 0)}
for name, (g, mode, start) in cases.items():
    ref, o_ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start, return_order=True)
    got = run(g, mode, start)
    deg = np.diff(g.row_ptr)
    if np.array_equal(got, ref):
        print(name, "ok", g.n, "maxdeg", deg.max()); continue
    o_got = got[::-1]
    i = int(np.nonzero(o_got != o_ref)[0][0])
    print(name, "MISMATCH at o-position", i, "of", g.n, "maxdeg", deg.max(), "got", o_got[i:i+5], "ref", o_ref[i:i+5],
          "deg got", deg[o_got[i:i+5]], "deg ref", deg[o_ref[i:i+5]], "is perm", len(set(got.tolist())) == g.n)
