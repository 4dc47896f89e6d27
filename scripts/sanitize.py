"""Small end-to-end run for compute-sanitizer: loopback P=2 Cora-shaped epoch,
an SpMM-first config (112 classes: the 32-lane CE row groups), a 1.5D loopback
epoch (MGGCN_F_REPL2, P = 4), a loopback P = 8 epoch with the default stage
groups and NaN-poisoned BC slots, dense-block epochs (tcgen05 blocks forced on small tiles: P = 1
and loopback P = 2, split groups + fix-up, widths 256 and 41), and the three GEMM ops (ragged shapes)."""
import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_icpp_balinsc22_b200 as mg
from paper_conf_icpp_balinsc22_b200 import GCN
for dims, P, n, m, c in (((1433, 16, 7), 2, 2708, 10556, 1), ((8, 128, 128, 112), 1, 3001, 60000, 1),
                         ((100, 64, 47), 4, 3001, 60000, 2), ((64, 48, 41), 8, 4001, 200000, 1)):
    rp, col = gen.rmat_csr(n, m, 5)
    X = gen.features(n, dims[0], 6); y = gen.labels(n, dims[-1], 7, 100)
    Ws = [gen.glorot(dims[l], dims[l + 1], 8 + l) for l in range(len(dims) - 1)]
    gm = GCN(n, rp, col, None, dims, P=P, perm_seed=9, loopback=P > 1, flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE,
             replicas=c)
    gm.set_weights(Ws)
    if P == 8:
        mg.mggcn_debug_poison(gm.m, 1)
    for host in (False, True):
        Xl, yl = gm.permute_rows(X), gm.permute_rows(y)
        Xin = Xl if host else torch.from_numpy(Xl).cuda()
        yin = yl if host else torch.from_numpy(yl).cuda()
        loss = gm.forward(Xin, yin, logits=torch.empty((c * n, dims[-1]), device="cuda"))
        gm.backward(); gm.step()
    print("epoch ok", dims, P, c, loss, flush=True)
    gm.close()
# dense blocks (dense.cu): forced on the small tiles of a 4096-vertex R-MAT (MGGCN_DENSE_* read at model creation)
os.environ.update(MGGCN_DENSE_THR="0.02", MGGCN_DENSE_MINFRAC="0", MGGCN_DENSE_MIN_ROWS="0", MGGCN_DENSE_MIN_ENTRIES="0")
for P in (1, 2):
    n, dims = 4096, (64, 256, 256, 41)
    rp, col = gen.rmat_csr(n, 400000, 17)
    X = gen.features(n, dims[0], 6); y = gen.labels(n, dims[-1], 7, 100)
    Ws = [gen.glorot(dims[l], dims[l + 1], 8 + l) for l in range(len(dims) - 1)]
    gm = GCN(n, rp, col, None, dims, P=P, perm_seed=9, loopback=P > 1, flags=mg.MGGCN_F_OVERLAP)
    assert mg.mggcn_dense_stats(gm.m)["blocks"] > 0
    gm.set_weights(Ws)
    Xl, yl = gm.permute_rows(X), gm.permute_rows(y)
    loss = gm.forward(torch.from_numpy(Xl).cuda(), torch.from_numpy(yl).cuda(), logits=torch.empty((n, dims[-1]), device="cuda"))
    gm.backward(); gm.step()
    print("dense epoch ok", P, loss, mg.mggcn_dense_stats(gm.m), flush=True)
    gm.close()
for k in ("MGGCN_DENSE_THR", "MGGCN_DENSE_MINFRAC", "MGGCN_DENSE_MIN_ROWS", "MGGCN_DENSE_MIN_ENTRIES"):
    os.environ.pop(k)
for op, (M, N, K) in ((0, (300, 41, 602)), (1, (257, 256, 41)), (2, (602, 47, 1000))):
    rng = np.random.default_rng(op)
    if op == 0: A, B = rng.standard_normal((M, 608)), rng.standard_normal((K, 48))
    elif op == 1: A, B = rng.standard_normal((M, 48)), rng.standard_normal((N, 48))
    else: A, B = rng.standard_normal((K, 608)), rng.standard_normal((K, 48))
    C = torch.zeros((M, (N + 7) // 8 * 8), device="cuda")
    mg.mggcn_debug_gemm(op, M, N, K, torch.tensor(A, dtype=torch.float32).cuda(), A.shape[1],
                        torch.tensor(B, dtype=torch.float32).cuda(), B.shape[1], C, C.shape[1])
    print("gemm ok", op, flush=True)
