"""One warm-up + N timed rcm_reorder calls on a config (for ncu captures)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import json
import torch, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
n_calls = int(sys.argv[2]) if len(sys.argv) > 2 else 2
g, mode, start = synth.config_graph(cfg)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
perm = torch.empty(g.n, dtype=torch.int32, device="cuda")
plan = rcm.Plan(g.n, g.nnz, **json.loads(os.environ.get("RCM_PLAN", "{}")))
for _ in range(n_calls):
    rcm.rcm_reorder(plan.handle, g.n, g.nnz, rp, ci, mode, start, perm)
print("status", rcm.rcm_sync_status(plan.handle))
