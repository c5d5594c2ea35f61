"""Time rcm_reorder_batched on full config 5 for the library in RCM_LIB (A/B sweeps).
Prints one JSON line: lib, ms (median of K), solo blocks, parity on 64 sampled matrices."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth, synth.device as sd, oracle
import paper_conf_ipps_mlakarwps21_b200 as rcm
K = int(sys.argv[1]) if len(sys.argv) > 1 else 5
b = sd.c5_generate(None, num=8192)
plan = rcm.Plan(b["total"], b["total_nnz"], flags=rcm.RCM_FLAG_BATCHED_ONLY, **json.loads(os.environ.get("RCM_PLAN", "{}")))
perm = torch.empty(b["total"], dtype=torch.int32, device="cuda")
def step():
    rcm.rcm_reorder_batched(plan.handle, 8192, b["total"], b["total_nnz"], b["node_off"], b["nnz_off"],
                            b["row_ptr_local"], b["col_idx_local"], rcm.RCM_START_MIN_DEGREE, None, perm)
for _ in range(2): step()
assert rcm.rcm_sync_status(plan.handle) == 0
ts = []
for _ in range(K):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); step(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
p = perm.cpu().numpy()
sizes = synth.c5_sizes(8192)
ok = 0
rng = np.random.default_rng(3)
sample = rng.choice(8192, 48, replace=False).tolist() + [int(np.argmax(sizes))]
for k in sample:
    g = synth.c5_matrix(k, int(sizes[k]))
    a0, a1 = int(b["node_off_h"][k]), int(b["node_off_h"][k + 1])
    ok += np.array_equal(p[a0:a1], oracle.rcm(g.row_ptr, g.col_idx, oracle.MIN_DEGREE))
splan = rcm.Plan(b["total"], b["total_nnz"], flags=rcm.RCM_FLAG_BATCHED_ONLY, collect_stats=1)
splan.reorder_batched(b["node_off"], b["nnz_off"], b["row_ptr_local"], b["col_idx_local"], b["total"], b["total_nnz"],
                      perm_local=perm)
st = splan.stats()
splan.close()
print(json.dumps({"lib": os.environ.get("RCM_LIB", "default"), "ms": round(statistics.median(ts), 3),
                  "batches": st["batches_executed"], "combined": st["overhang_forwards"],
                  "min_ms": round(min(ts), 3), "solo_blocks": plan.info()["solo_blocks"],
                  "parity_sample": f"{ok}/{len(sample)}"}), flush=True)
