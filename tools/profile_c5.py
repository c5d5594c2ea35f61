"""Warm-up + N rcm_reorder_batched calls on (a prefix of) config 5, for ncu.
usage: python tools/profile_c5.py [num_mats=8192] [calls=2]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import synth.device as sd  # noqa: E402
import paper_conf_ipps_mlakarwps21_b200 as rcm  # noqa: E402

num = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
calls = int(sys.argv[2]) if len(sys.argv) > 2 else 2
mats = np.arange(num) if num == 8192 else np.random.default_rng(1).choice(8192, num, replace=False)
b = sd.c5_generate(np.sort(mats), num=8192)
plan = rcm.Plan(b["total"], b["total_nnz"], flags=rcm.RCM_FLAG_BATCHED_ONLY, **(eval(os.environ.get("RCM_PLAN", "{}"))))
perm = torch.empty(b["total"], dtype=torch.int32, device="cuda")
for _ in range(calls):
    rcm.rcm_reorder_batched(plan.handle, len(mats), b["total"], b["total_nnz"], b["node_off"], b["nnz_off"],
                            b["row_ptr_local"], b["col_idx_local"], rcm.RCM_START_MIN_DEGREE, None, perm)
print("status", rcm.rcm_sync_status(plan.handle))
