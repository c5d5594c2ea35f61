#!/bin/bash
# GL finder timing (rcm_find_pseudo_peripheral from the max-degree node) on C2-C4, current vs LIB
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
cat > /tmp/gl_time.py <<'PY'
import os, sys, statistics, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth, oracle
import paper_conf_ipps_mlakarwps21_b200 as rcm
for cfg in (2, 3, 4):
    g, _, _ = synth.config_graph(cfg)
    s0 = int(np.argmax(np.diff(g.row_ptr)))
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    plan = rcm.Plan(g.n, g.nnz)
    out = torch.empty(1, dtype=torch.int32, device="cuda")
    ts = []
    for i in range(6):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); rcm.rcm_find_pseudo_peripheral(plan.handle, g.n, g.nnz, rp, ci, s0, out); e1.record()
        torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    ok = int(out.item()) == oracle.gl(g.row_ptr, g.col_idx, s0)
    print(json.dumps({"lib": os.environ.get("RCM_LIB", "default"), "cfg": cfg, "ms": round(statistics.median(ts[2:]), 3), "ok": ok}), flush=True)
    plan.close()
PY
timeout 600 python /tmp/gl_time.py > gpurun_out/gl_default.jsonl 2> gpurun_out/gl.err
RCM_LIB=build/librcm_${LIB}.so timeout 600 python /tmp/gl_time.py > gpurun_out/gl_${LIB}.jsonl 2>> gpurun_out/gl.err
