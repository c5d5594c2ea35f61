"""Per-slot event trace of one reorder (collect_stats=3) -> critical generation
chain and per-stage latencies along it."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm
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
buf = (ctypes.c_ulonglong * (8 * cnt))()
lib.rcm_debug_trace(plan.handle, cnt, buf)
tr = np.frombuffer(buf, dtype=np.uint64).reshape(cnt, 8).astype(np.int64)
real = np.nonzero(tr[:, 0])[0]
t0 = tr[real, 0].min()
ev = (tr[real, :7] - t0) / 1000.0          # us
gen = (tr[real, 7] >> 32)
print("slots traced", len(real), "span us", round(ev[:, 6].max(), 1))
names = ["discover", "wait_D", "redisc+agg", "wait_C", "output", "generate"]
d = np.diff(ev[:, :7], axis=1)
print("mean per-slot us:", {n: round(float(np.mean(d[:, i])), 2) for i, n in enumerate(names)})
# critical generation chain from the slot that published last
slot_to_row = {int(s): i for i, s in enumerate(real)}
cur = int(real[np.argmax(ev[:, 6])])
chain = []
while cur in slot_to_row:
    chain.append(cur)
    gsl = int(tr[cur, 7] >> 32)
    if cur == 0 or gsl == cur or (tr[cur, 7] == 0 and cur != 0):
        break
    cur = gsl
chain = chain[::-1]
print("chain depth", len(chain))
rows = [slot_to_row[s] for s in chain]
pick = []
for a, b in zip(rows[:-1], rows[1:]):
    pick.append(ev[b, 0] - ev[a, 6])
dd = d[rows]
print("along chain mean us:", {n: round(float(np.mean(dd[:, i])), 2) for i, n in enumerate(names)},
      "pickup(after parent's gen end)", round(float(np.mean(pick)), 2) if pick else None)
print("chain total us", round(ev[rows[-1], 6] - ev[rows[0], 0], 1))
