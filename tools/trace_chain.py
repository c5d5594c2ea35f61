"""Per-slot event trace of one reorder (collect_stats=3, RCM_TRACE build) ->
critical generation chain and per-stage latencies along it.

Events per slot (rcm_batch.cuh kTraceW): 0 dequeued, 1 parents loaded,
2 discovered, 3 Discovered known, 4 aggregate published, 5 before prefix,
6 prefix known, 7 output written, 8 batches published, 9 slot claimed,
15 generator slot << 32 | block."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm
W = 16
lib = rcm._load()
lib.rcm_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_ulonglong)]
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
opts = eval(sys.argv[2]) if len(sys.argv) > 2 else {}
g, mode, start = synth.config_graph(cfg)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
plan = rcm.Plan(g.n, g.nnz, collect_stats=3, **opts)
for _ in range(3):
    perm = plan.reorder(rp, ci, mode, start)
st = plan.stats()
cnt = min(st["batches_generated"] + 2, 1 << 20)
buf = (ctypes.c_ulonglong * (W * cnt))()
lib.rcm_debug_trace(plan.handle, cnt, buf)
tr = np.frombuffer(buf, dtype=np.uint64).reshape(cnt, W).astype(np.int64)
if len(sys.argv) > 3:
    np.save(sys.argv[3], tr)   # raw trace for offline analysis
real = np.nonzero(tr[:, 0])[0]
t0 = tr[real, 0].min()
ev = (tr[real, :10] - t0) / 1000.0          # us
print("slots traced", len(real), "span us", round(ev[:, 8].max(), 1))
names = ["parents", "discover", "wait_D", "redisc+agg", "sort/-", "wait_C", "output", "generate"]
d = np.diff(ev[:, :9], axis=1)
print("mean per-slot us:", {n: round(float(np.mean(d[:, i])), 2) for i, n in enumerate(names)})
slot_to_row = {int(s): i for i, s in enumerate(real)}
cur = int(real[np.argmax(ev[:, 8])])
chain = []
while cur in slot_to_row:
    chain.append(cur)
    gsl = int(tr[cur, W - 1] >> 32)
    if cur == 0 or gsl == cur or (tr[cur, W - 1] == 0 and cur != 0):
        break
    cur = gsl
chain = chain[::-1]
print("chain depth", len(chain))
rows = [slot_to_row[s] for s in chain]
pick, claim_late = [], []
for a, b in zip(rows[:-1], rows[1:]):
    pick.append(ev[b, 0] - ev[a, 8])
    claim_late.append(max(0.0, ev[b, 9] - ev[a, 8]))   # slot claimed only after it was published
dd = d[rows]
print("along chain mean us:", {n: round(float(np.mean(dd[:, i])), 2) for i, n in enumerate(names)},
      "pickup", round(float(np.mean(pick)), 2) if pick else None,
      "of which no free block", round(float(np.mean(claim_late)), 2) if pick else None)
# batch sizes along the chain vs overall
sizes = None
hq = [int(tr[s, 10]) - int(tr[s, 11]) for s in chain]
print("head - q_off at chain publishes: median", int(np.median(hq)), "min", min(hq), "max", max(hq))
print("chain total us", round(ev[rows[-1], 8] - ev[rows[0], 0], 1))
# in-flight slots (claimed, not finished) sampled at every chain publish
fin = ev[:, 8]; clm = ev[:, 9]
inflight = [int(np.sum((clm <= ev[r, 8]) & (fin > ev[r, 8]))) for r in rows]
print("in-flight slots at chain publishes: median", int(np.median(inflight)), "max", max(inflight))
