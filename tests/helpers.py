"""Small-graph builders and independent dense references used by the tests."""
import json
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def fp32_third():
    return np.float32(1.0) / np.float32(3.0)


def golden_val(x):
    """Golden files write 1/3 as the string "1/3" (fp32 division)."""
    if isinstance(x, str):
        a, b = x.split("/")
        return np.float32(np.float32(float(a)) / np.float32(float(b)))
    return np.float32(x)


def csr_from_edges(n, edges, vals=None):
    """CSR (rowptr int64, col int32, vals or None) sorted by (row, col), stable for duplicates."""
    edges = list(edges)
    order = sorted(range(len(edges)), key=lambda e: (edges[e][0], edges[e][1], e))
    rowptr = np.zeros(n + 1, dtype=np.int64)
    for u, _ in edges:
        rowptr[u + 1] += 1
    rowptr = np.cumsum(rowptr)
    col = np.array([edges[e][1] for e in order], dtype=np.int32)
    v = None if vals is None else np.array([vals[e] for e in order], dtype=np.float32)
    return rowptr, col, v


def dense_ahat(n, rowptr, col, vals=None):
    """Dense fp64 Â with Â[u, v] = A_uv / sum_w A_wv (Eq. 2), duplicates summed."""
    A = np.zeros((n, n))
    for u in range(n):
        for e in range(rowptr[u], rowptr[u + 1]):
            A[u, col[e]] += 1.0 if vals is None else float(vals[e])
    deg = A.sum(axis=0)
    with np.errstate(invalid="ignore", divide="ignore"):
        Ah = np.where(deg[None, :] > 0, A / np.where(deg > 0, deg, 1)[None, :], 0.0)
    return Ah


def perm_matrix(perm):
    n = perm.shape[0]
    Pm = np.zeros((n, n))
    Pm[perm, np.arange(n)] = 1.0      # (Pm x)[perm[v]] = x[v]
    return Pm


def random_graph(n, m, seed):
    import gen
    rp, col = gen.rmat_csr(n, m, seed)
    return rp, col


def random_directed(n, m, seed, weighted=False, dup=True):
    """Random directed multigraph (not symmetric), optional positive weights."""
    rng = np.random.default_rng(seed)
    u = rng.integers(0, n, m)
    v = rng.integers(0, n, m)
    if not dup:
        key = np.unique(u * n + v)
        u, v = key // n, key % n
    edges = list(zip(u.tolist(), v.tolist()))
    vals = rng.uniform(0.5, 2.0, len(edges)).astype(np.float32).tolist() if weighted else None
    return csr_from_edges(n, edges, vals)


def torch_epoch(Ah_perm, Xp, yp, Ws, relu_last=False):
    """Textbook dense GCN (Eq. 1-4) in torch float64 with autograd.
    Returns (logits, loss, grads)."""
    import torch
    A = torch.tensor(Ah_perm, dtype=torch.float64)
    H = torch.tensor(Xp, dtype=torch.float64)
    Wt = [torch.tensor(W, dtype=torch.float64, requires_grad=True) for W in Ws]
    L = len(Ws)
    for l in range(L):
        Z = A.T @ H @ Wt[l]
        H = torch.relu(Z) if (l < L - 1 or relu_last) else Z
    y = torch.tensor(yp, dtype=torch.int64)
    ntrain = int((y >= 0).sum())
    loss = torch.nn.functional.cross_entropy(H, y.clamp(min=0), reduction="none")
    loss = (loss * (y >= 0)).sum() / ntrain
    loss.backward()
    return H.detach().numpy(), float(loss), [w.grad.numpy() for w in Wt]
