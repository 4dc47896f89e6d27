"""Multi-process plumbing around the C ABI (one process per GPU).

torch.distributed only carries the 128-byte ncclUniqueId (the library builds
its own NCCL communicator, because torch does not expose its ncclComm_t) or
the 128-byte CUDA-IPC descriptors of the MGGCN_F_IPC backend, and the
max-over-ranks timing.  All data movement of the hot path is inside the
library (P-stage broadcasts, W_G all-reduce).
"""
from __future__ import annotations


def share_nccl_id(dist, make_id):
    """Rank 0 creates the id with `make_id()`; every rank returns the same 128 bytes."""
    obj = [make_id() if dist.get_rank() == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    return obj[0]


def ipc_exchange(dist):
    """Returns f(blob) -> the P MGGCN_F_IPC blobs in rank order (all_gather over `dist`)."""
    def f(blob):
        out = [None] * dist.get_world_size()
        dist.all_gather_object(out, blob)
        return out
    return f


def local_rows(perm, p, rank, M):
    """Rows p(rank)..p(rank+1)-1 of the permuted matrix M' (M'[perm[v]] = M[v])."""
    import numpy as np
    M = np.asarray(M)
    inv = np.empty_like(perm)
    inv[perm] = np.arange(perm.shape[0])
    return np.ascontiguousarray(M[inv[p[rank]:p[rank + 1]]])


def max_over_ranks(dist, value, device=None):
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
