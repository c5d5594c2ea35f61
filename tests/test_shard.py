"""Multi-rank host logic of the config-5 path on CPU (gloo, world_size 2):
deterministic LPT partition, per-rank work, grouped point-to-point gather to
rank 0, reassembly in global matrix order."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_mlakarwps21_b200 import shard


def test_lpt_partition_is_deterministic_and_complete():
    w = np.random.default_rng(0).integers(1, 1000, 101)
    p1 = shard.lpt_partition(w, 4)
    p2 = shard.lpt_partition(w.copy(), 4)
    assert p1 == p2
    assert sorted(sum(p1, [])) == list(range(101))
    loads = [int(w[p].sum()) for p in p1]
    assert max(loads) - min(loads) <= int(w.max())


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    import oracle
    import synth
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    b = synth.c5_batch(num=9, seed=5, lo=40, hi=400)
    nnz = np.diff(b.nnz_off)
    n = np.diff(b.node_off)
    parts = shard.lpt_partition(nnz, world)
    # this rank's share (the GPU path would call rcm_reorder_batched here)
    mine = [oracle.rcm(b.row_ptr_local[b.node_off[k] + k: b.node_off[k + 1] + k + 1],
                       b.col_idx_local[b.nnz_off[k]: b.nnz_off[k + 1]], oracle.MIN_DEGREE) for k in parts[rank]]
    local = torch.from_numpy(np.concatenate(mine).astype(np.int32))
    sizes = [int(n[p].sum()) for p in parts]
    got = shard.gather_to_root(local, sizes, rank, world)
    if rank == 0:
        per = shard.assemble([g.numpy() for g in got], parts, n)
        ref = oracle.rcm_batched(b.node_off, b.nnz_off, b.row_ptr_local, b.col_idx_local, oracle.MIN_DEGREE)
        q.put(bool(np.array_equal(np.concatenate(per), ref)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gather_ranks_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=120)
    assert all(p.exitcode == 0 for p in procs)
    assert q.get(timeout=5) is True
