"""Per-round timeline of the leveled traversal (RCM_FLAG_LEVELED, collect_stats=3),
block 0's view per round: R, barrier 1, W (prefix + output), D, level barrier (us).
usage: python tools/trace_leveled.py <cfg> [opts-dict]"""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm
W = 16
lib = rcm._load()
lib.rcm_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_ulonglong)]
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
opts = eval(sys.argv[2]) if len(sys.argv) > 2 else {}
opts.setdefault("flags", 32)
g, mode, start = synth.config_graph(cfg)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
plan = rcm.Plan(g.n, g.nnz, collect_stats=3, **opts)
for _ in range(3):
    perm = plan.reorder(rp, ci, mode, start)
cnt = 1 << 16
buf = (ctypes.c_ulonglong * (W * cnt))()
lib.rcm_debug_trace(plan.handle, cnt, buf)
tr = np.frombuffer(buf, dtype=np.uint64).reshape(cnt, W).astype(np.int64)
rows = np.nonzero(tr[:, 0])[0]
tr = tr[rows]
nxt = np.append(tr[1:, 0], tr[-1, 4])
end = np.where(tr[:, 5] > 0, tr[:, 5], nxt)
ph = {"R": tr[:, 1] - tr[:, 0], "bar1": tr[:, 2] - tr[:, 1], "W": tr[:, 3] - tr[:, 2], "D": tr[:, 4] - tr[:, 3],
      "bar2": end - tr[:, 4]}
# barrier split (rows with a level barrier): wait for the last block vs release latency
lvl = tr[:, 5] > 0
ph["b1_wait_last"] = tr[:, 6] - tr[:, 1]
ph["b1_release"] = tr[:, 2] - tr[:, 6]
ph["b2_wait_last"] = np.where(lvl, tr[:, 7] - tr[:, 4], 0)
ph["b2_release"] = np.where(lvl, tr[:, 5] - tr[:, 7], 0)
tot = {k: round(float(v.sum()) / 1000, 1) for k, v in ph.items()}
print(json.dumps({"cfg": cfg, "rounds": len(tr), "levels": int(tr[:, 9].max()) + 1 if len(tr) else 0,
                  "span_us": round(float(end[-1] - tr[0, 0]) / 1000, 1), "sum_us": tot,
                  "mean_us": {k: round(float(v.mean()) / 1000, 2) for k, v in ph.items()}}))
big = np.argsort(-tr[:, 8])[:8]
for i in sorted(big):
    print(json.dumps({"round": int(i), "level": int(tr[i, 9]), "children": int(tr[i, 8]), "max_block": int(tr[i, 10]),
                      **{k: round(float(v[i]) / 1000, 2) for k, v in ph.items()}}))
