import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_ipps_mlakarwps21_b200 as rcm
g, mode, start = synth.config_graph(4, "small")
ref, o_ref = oracle.rcm(g.row_ptr, g.col_idx, mode, start, return_order=True)
deg = np.diff(g.row_ptr)
for cs in (0, 1):
    for ip in (False, True):
        bad = 0
        for it in range(30):
            plan = rcm.Plan(g.n, g.nnz, solo_threshold=g.n, collect_stats=cs)
            iperm = torch.empty(g.n, dtype=torch.int32, device="cuda") if ip else None
            got = plan.reorder(torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda(), mode, start, iperm=iperm).cpu().numpy()
            st = plan.stats()
            plan.close()
            if not np.array_equal(got, ref):
                bad += 1
                o_got = got[::-1]
                i = int(np.nonzero(o_got != o_ref)[0][0])
                if bad <= 2:
                    print("cs", cs, "ip", ip, "MISMATCH at", i, o_got[max(0,i-3):i+4], o_ref[max(0,i-3):i+4], deg[o_got[i:i+4]], deg[o_ref[i:i+4]], st)
        print("cs", cs, "iperm", ip, "bad", bad, "of 30")
