"""Multi-GPU plumbing for independent matrices (config 5):
a deterministic LPT partition of matrices over ranks and the gather of the
per-rank permutations into rank 0 with grouped point-to-point transfers
(NCCL over NVLink on the GPU box; gloo in the CPU tests).  The traversal
itself never crosses a device boundary."""
from __future__ import annotations

import numpy as np


def lpt_partition(weights, parts: int):
    """Longest-processing-time first: heaviest matrix to the least-loaded rank;
    ties by index, so every rank computes the same partition."""
    w = np.asarray(weights, dtype=np.int64)
    order = np.lexsort((np.arange(w.size), -w))
    load = np.zeros(parts, np.int64)
    out = [[] for _ in range(parts)]
    for i in order:
        p = int(np.argmin(load))
        out[p].append(int(i))
        load[p] += int(w[i])
    return [sorted(o) for o in out]


def gather_to_root(local, part_sizes, rank: int, world: int, root: int = 0):
    """Rank `root` receives every rank's 1-D tensor (sizes part_sizes[r]) into a
    list; other ranks send theirs.  One batched isend/irecv group (the NCCL
    ncclGroupStart / Send / Recv / ncclGroupEnd pattern)."""
    import torch
    import torch.distributed as dist
    if world == 1:
        return [local]
    # NCCL moves device tensors over NVLink; gloo (CPU tests, harness checks)
    # moves host copies
    host = dist.get_backend() != "nccl" and local.is_cuda
    buf = local.cpu() if host else local
    if rank == root:
        out = [buf if r == root else torch.empty(part_sizes[r], dtype=local.dtype, device=buf.device)
               for r in range(world)]
        ops = [dist.P2POp(dist.irecv, out[r], r) for r in range(world) if r != root]
    else:
        out = None
        ops = [dist.P2POp(dist.isend, buf, root)]
    for w in dist.batch_isend_irecv(ops):
        w.wait()
    if host and out is not None:
        out = [o.to(local.device) for o in out]
    return out


def assemble(gathered, parts, node_counts):
    """Concatenated per-rank permutations -> list of per-matrix local perms in
    global matrix order."""
    res = [None] * len(node_counts)
    for r, mats in enumerate(parts):
        buf = gathered[r]
        off = 0
        for k in mats:
            n = int(node_counts[k])
            res[k] = buf[off:off + n]
            off += n
    return res
