"""Per-stage SM cycles of the chain workers (collect_stats=2), Fig. 6 analogue."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm
for cfg in [int(c) for c in (sys.argv[1:] or ["2"])]:
    g, mode, start = synth.config_graph(cfg)
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    for opts in (dict(collect_stats=2), dict(collect_stats=1)):
        plan = rcm.Plan(g.n, g.nnz, **opts, **json.loads(os.environ.get("RCM_PLAN", "{}")))
        for _ in range(3): plan.reorder(rp, ci, mode, start)
        st = plan.stats(); tm = plan.timing(); info = plan.info()
        cyc = st.get("stage_cycles", {})
        tot = sum(cyc.values()) or 1
        print(json.dumps({"cfg": cfg, "opts": opts, "timing": {k: round(v, 3) for k, v in tm.items()},
                          "stages_pct": {k: round(100 * v / tot, 1) for k, v in cyc.items()},
                          "cycles_per_batch": round(tot / max(1, st["batches_executed"])),
                          "stats": {k: v for k, v in st.items() if k != "stage_cycles"}, "plan": info}), flush=True)
        plan.close()
