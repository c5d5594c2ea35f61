"""Per-slot event trace (RCM_TRACE build, collect_stats=3) -> time-binned
occupancy of the persistent blocks by state, for one reorder of a config.

States of a claimed slot (events, rcm_batch.cuh kTraceW):
  wait_pub [9,0)  claimed, descriptor not yet published
  work_a   [0,2)  parents + speculative discovery
  wait_D   [2,3)  (speculative sort +) waiting for predecessors' discovery
  redisc   [3,4)  rediscovery + count (+ AGG publish)
  sort     [4,5)  sort after early rediscovery
  wait_C   [5,6)  prefix look-back
  work_b   [6,8)  output + generation + publish"""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm
W = 16
lib = rcm._load()
lib.rcm_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_ulonglong)]
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
opts = eval(sys.argv[2]) if len(sys.argv) > 2 else {}
nbins = int(sys.argv[3]) if len(sys.argv) > 3 else 20
g, mode, start = synth.config_graph(cfg)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
plan = rcm.Plan(g.n, g.nnz, collect_stats=3, **opts)
for _ in range(3):
    perm = plan.reorder(rp, ci, mode, start)
st = plan.stats(); info = plan.info()
cnt = min(st["batches_generated"] + 2, 1 << 20)
buf = (ctypes.c_ulonglong * (W * cnt))()
lib.rcm_debug_trace(plan.handle, cnt, buf)
tr = np.frombuffer(buf, dtype=np.uint64).reshape(cnt, W).astype(np.int64)
real = np.nonzero((tr[:, 0] != 0) & (tr[:, 8] != 0))[0]
ev = tr[real, :10].astype(np.float64)
t0 = ev[:, 0].min()
ev = (ev - t0) / 1000.0
ev[ev < -1e6] = np.nan
span = np.nanmax(ev[:, 8])
nb = info["blocks"]
print(f"cfg {cfg} opts {opts} blocks {nb} slots {len(real)} span_us {span:.1f}")
states = [("wait_pub", 9, 0), ("work_a", 0, 2), ("wait_D", 2, 3), ("redisc", 3, 4), ("sort", 4, 5),
          ("wait_C", 5, 6), ("work_b", 6, 8)]
edges = np.linspace(0, span, nbins + 1)
rows = []
for b in range(nbins):
    lo, hi = edges[b], edges[b + 1]
    row = {}
    for name, a, z in states:
        s, e = ev[:, a], ev[:, z]
        ok = np.isfinite(s) & np.isfinite(e) & (e >= s)
        ov = np.clip(np.minimum(e[ok], hi) - np.maximum(s[ok], lo), 0, None)
        row[name] = float(ov.sum() / (hi - lo))
    row["busy"] = sum(row.values())
    row["done_batches"] = int(np.sum((ev[:, 8] >= lo) & (ev[:, 8] < hi)))
    rows.append(row)
hdr = "bin  t_us   " + " ".join(f"{n:>8s}" for n, _, _ in states) + "  sum/blk  batches"
print(hdr)
for b, row in enumerate(rows):
    print(f"{b:3d} {edges[b]:6.0f}  " + " ".join(f"{row[n]:8.1f}" for n, _, _ in states) +
          f"  {row['busy'] / nb:7.2f}  {row['done_batches']:7d}")
tot = {n: float(np.nansum(np.clip(ev[:, z] - ev[:, a], 0, None))) for n, a, z in states}
T = sum(tot.values())
print("share of slot time:", {k: round(100 * v / T, 1) for k, v in tot.items()})
print("mean per slot us:", {k: round(v / len(real), 2) for k, v in tot.items()})
