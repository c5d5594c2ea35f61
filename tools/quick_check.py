"""Quick GPU sanity run: tiny graphs through every path, then configs."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import torch
import oracle, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm

import ctypes
_lib = rcm._load()
_lib.rcm_debug_info.argtypes = [ctypes.c_void_p, ctypes.POINTER(ctypes.c_longlong)]

def run(g, mode, start, **opts):
    plan = rcm.Plan(max(g.n, 1), max(g.nnz, 1), collect_stats=1, **opts)
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    try:
        perm = plan.reorder(rp, ci, mode, start).cpu().numpy()
    except Exception as e:
        a = (ctypes.c_longlong * 8)()
        _lib.rcm_debug_info(plan.handle, a)
        return None, str(e) + " dbg=" + str(list(a)) + " stats=" + str(plan.stats())
    st = plan.stats(); plan.close()
    return perm, st

tiny = [("path7", synth.path(7)), ("star12", synth.star(12)), ("grid7x5", synth.grid2d(7, 5)),
        ("gnp80", synth.gnp(80, 0.05, 1)), ("union", synth.disjoint_union([synth.path(4), synth.star(30), synth.path(1)])),
        ("g3d", synth.relabel(synth.grid3d_27(7, 6, 5), synth.randperm(210, 3)))]
paths = {"solo": {}, "chain": dict(flags=8, solo_threshold=-1), "chain_bs1": dict(flags=8, solo_threshold=-1, batch_nodes=1)}
which = sys.argv[1:] or ["tiny", "small", "full"]
if "tiny" in which:
    for pname, opts in paths.items():
        for name, g in tiny:
            for mode, start in [(0, g.n // 2), (1, 0)]:
                ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
                t = time.time()
                got, st = run(g, mode, start, **opts)
                ok = got is not None and np.array_equal(got, ref)
                print(f"{pname:10s} {name:8s} mode={mode} ok={ok} t={time.time()-t:.2f}s", "" if ok else st, flush=True)
if "small" in which:
    for cfg in [1, 2, 3, 4]:
        g, mode, start = synth.config_graph(cfg, "small")
        ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
        for pname, opts in [("solo", dict(solo_threshold=g.n)), ("chain", dict(solo_threshold=-1))]:
            t = time.time(); got, st = run(g, mode, start, **opts)
            ok = got is not None and np.array_equal(got, ref)
            print(f"small C{cfg} {pname} ok={ok} t={time.time()-t:.2f}s {st}", flush=True)
if "full" in which:
    for cfg in [1, 2, 4, 3]:
        g, mode, start = synth.config_graph(cfg)
        ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
        t = time.time(); got, st = run(g, mode, start)
        ok = got is not None and np.array_equal(got, ref)
        print(f"full C{cfg} ok={ok} t={time.time()-t:.2f}s {st}", flush=True)
