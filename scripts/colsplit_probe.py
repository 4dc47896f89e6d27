"""Probe: does splitting the gathered operand into K column blocks (each
processed over all rows, accumulating) raise the SpMM's gather rate enough to
pay for the extra passes?  Times mggcn_debug_spmm on Reddit-shaped column
sub-graphs (permuted ids, identity perm inside the library)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402
from paper_conf_icpp_balinsc22_b200 import GCN  # noqa: E402

w = gen.WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "reddit"]
width = int(sys.argv[2]) if len(sys.argv) > 2 else 256
n = w.n
rp, col = gen.rmat_csr(n, w.m, w.seed_G)
perm = np.random.default_rng(5).permutation(n)
u = perm[np.repeat(np.arange(n), np.diff(rp))]
v = perm[col.astype(np.int64)]
# sort by (u, v) once
o = np.lexsort((v, u))
u, v = u[o], v[o]
B = torch.randn((n, width), device="cuda")
out = torch.empty((n, width), device="cuda")


def time_graph(uu, vv):
    rpk = np.zeros(n + 1, np.int64)
    np.add.at(rpk, uu + 1, 1)
    rpk = np.cumsum(rpk)
    gm = GCN(n, rpk, vv.astype(np.int32), None, (width, width), perm_seed=0,
             flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
    mg.mggcn_debug_spmm(gm.m, 1, B, width, width, out, width)
    torch.cuda.synchronize()
    gm.profile(reset=True)
    for _ in range(5):
        mg.mggcn_debug_spmm(gm.m, 1, B, width, width, out, width)
    torch.cuda.synchronize()
    ms, cnt = gm.profile(reset=True)["spmm"]
    gm.close()
    return ms / 5


for K in (1, 2, 4, 8):
    bounds = [n * k // K for k in range(K + 1)]
    tot = 0.0
    parts = []
    for k in range(K):
        sel = (v >= bounds[k]) & (v < bounds[k + 1])
        t = time_graph(u[sel], v[sel])
        parts.append(round(t, 3))
        tot += t
    print(f"K={K}: total {tot:.3f} ms  parts {parts}", flush=True)
