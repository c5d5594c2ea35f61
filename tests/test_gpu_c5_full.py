"""GPU: bit-identity on the FULL config 5 (all 8,192 mesh matrices, ~176 M
nodes, ~2.67 G nnz), the north star's "identical on all five configs" for the
batched path.  The batch is generated on the device (synth.device, bit-identical
to synth.c5_matrix), reordered with rcm_reorder_batched in the configuration
bench.py times, copied back, and every matrix is compared with the serial
oracle (oracle.rcm_batched on all host cores, matrices are independent).  The
device-side generator itself is checked against the numpy generator on sampled
matrices (test_gpu_parity.test_c5_device_generator_matches_numpy)."""
import os

import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def test_full_c5_bit_identical():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import synth.device as sd
    import paper_conf_ipps_mlakarwps21_b200 as rcm
    b = sd.c5_generate(None, num=8192)
    plan = rcm.Plan(b["total"], b["total_nnz"])
    perm = plan.reorder_batched(b["node_off"], b["nnz_off"], b["row_ptr_local"], b["col_idx_local"],
                                b["total"], b["total_nnz"]).cpu().numpy()
    plan.close()
    rp = b["row_ptr_local"].cpu().numpy()
    ci = b["col_idx_local"].cpu().numpy()
    node_off, nnz_off = b["node_off_h"], b["nnz_off_h"]
    del b
    torch.cuda.empty_cache()
    ref = oracle.rcm_batched(node_off, nnz_off, rp, ci, oracle.MIN_DEGREE, threads=os.cpu_count() or 1)
    bad = [k for k in range(8192) if not np.array_equal(perm[node_off[k]:node_off[k + 1]],
                                                       ref[node_off[k]:node_off[k + 1]])]
    assert not bad, f"{len(bad)} of 8192 matrices differ, first {bad[:10]}"
