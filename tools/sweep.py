"""Time rcm_reorder on one config for a grid of plan options (L2 flushed per step)."""
import itertools, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth, oracle
import paper_conf_ipps_mlakarwps21_b200 as rcm

def main():
    cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    grid = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [{}]
    steps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
    g, mode, start = synth.config_graph(cfg)
    ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start)
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for opts in grid:
        plan = rcm.Plan(g.n, g.nnz, **opts)
        perm = torch.empty(g.n, dtype=torch.int32, device="cuda")
        for _ in range(2):
            rcm.rcm_reorder(plan.handle, g.n, g.nnz, rp, ci, mode, start, perm)
        ts = []
        for _ in range(steps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); rcm.rcm_reorder(plan.handle, g.n, g.nnz, rp, ci, mode, start, perm); e1.record()
            torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
        st = rcm.rcm_sync_status(plan.handle)
        ok = np.array_equal(perm.cpu().numpy(), ref)
        ph = plan.timing(); info = plan.info(); plan.close()
        sp = rcm.Plan(g.n, g.nnz, collect_stats=2, **opts); sp.reorder(rp, ci, mode, start); stt = sp.stats(); sp.close()
        cyc = stt.get("stage_cycles", {}); tot = max(1, sum(cyc.values()))
        print(json.dumps({"cfg": cfg, "opts": opts, "ms_med": round(float(np.median(ts)), 4), "ms_min": round(min(ts), 4),
                          "ok": ok, "status": st, "phases": {k: round(v, 3) for k, v in ph.items()},
                          "T": info["temp_elems"], "blocks": info["blocks"],
                          "exec": stt["batches_executed"], "empty": stt["batches_empty"], "fwd": stt["overhang_forwards"],
                          "late": stt["rediscover_late"], "early": stt["rediscover_early"],
                          "removed": stt["candidates_removed"], "spec": stt["candidates_speculative"],
                          "oversize": stt["oversize_batches"], "solo": stt["solo_problems"], "comps": stt["components"],
                          "stage_pct": {k: round(100 * v / tot, 1) for k, v in cyc.items()}}), flush=True)

main()
