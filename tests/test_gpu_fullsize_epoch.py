"""Step-by-step parity of ONE WHOLE EPOCH at BASELINE.json's full sizes, in
the launch configuration bench.py times (P = 1, overlap + profiling, device
inputs in the padded layout, coalesced tiles).

The oracle cannot run a full epoch at these sizes in seconds (≈ 440 s of one
core for Reddit), so every step of the GPU epoch is checked against the
oracle applied to the GPU's own inputs of that step (read back with
mggcn_debug_layer):
  forward   Z_l = Â'^T H_l W_l on sampled rows (Eq. 5-7), ReLU;
  loss      softmax-CE of the GPU logits, full;
  backward  W_G,l = H_l^T (Â' Z_G,l) on sampled columns (Eq. 9-10, C2), or
            T_0^T Z_G,0 for an SpMM-first layer 0 (§4.4, C11);
            Z_G,l-1 = (Â' Z_G,l) W_l^T ⊙ 1[H_l > 0] on sampled rows (Eq. 8, 11);
  Adam      the oracle's update of the GPU's W_G (C6).
Each check's tolerance is north_star's 1e-3 (relative to the sample's max)."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu
REL_TOL = 1e-3


def rel(x, r):
    return float(np.abs(np.asarray(x, np.float64) - r).max() / max(np.abs(r).max(), 1e-30))


@pytest.mark.parametrize("name", ["reddit", "proteins", "products"])
def test_fullsize_epoch_stepwise(name):
    assert torch.cuda.is_available()
    import paper_conf_icpp_balinsc22_b200 as mg
    from paper_conf_icpp_balinsc22_b200 import GCN
    w = gen.WORKLOADS[name]
    dims, L = w.dims, len(w.dims) - 1
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    X = gen.features(w.n, dims[0], w.seed_X)
    y = gen.labels(w.n, dims[-1], w.seed_y)
    Ws = [gen.glorot(dims[l], dims[l + 1], w.seed_W + l) for l in range(L)]
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    order = ["S" if oracle.spmm_first(dims[l], dims[l + 1]) else "G" for l in range(L)]

    gm = GCN(w.n, rp, col, None, dims, perm_seed=w.perm_seed, flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
    try:
        assert np.array_equal(gm.perm, pg.perm)
        gm.set_weights(Ws)
        Xp, yp = gm.permute_rows(X), gm.permute_rows(y)
        del X
        Xd, yd = gm.device_inputs(Xp), torch.from_numpy(yp).cuda()
        logits = torch.empty((w.n, dims[-1]), dtype=torch.float32, device="cuda")
        loss = gm.forward(Xd, yd, want_loss=True, logits=logits)
        H = [Xp] + [mg.mggcn_debug_layer(gm.m, l, (w.n, dims[l + 1])) for l in range(L - 1)]
        Zlast = logits.cpu().numpy()

        # sampled rows: the biggest hub (split rows + fix-up), a zero-in-degree vertex, 62 random
        deg = np.diff(rp)
        rng = np.random.default_rng(7)
        R = np.unique(np.array([int(pg.perm[np.argmax(deg)]), int(pg.perm[np.argmin(deg)])] +
                               rng.choice(w.n, 62, replace=False).tolist(), np.int64))

        # ---- forward, layer by layer from the GPU's H_l
        for l in range(L):
            Zs = oracle.gemm(oracle.spmm(pg.At, H[l], rows=R).astype(np.float64), Ws[l].astype(np.float64))
            got = H[l + 1][R] if l < L - 1 else Zlast[R]
            ref = oracle.relu(Zs) if l < L - 1 else Zs
            assert rel(got, ref) < REL_TOL, ("forward", l, rel(got, ref))

        # ---- loss and its gradient from the GPU logits
        ntrain = int((yp >= 0).sum())
        lsum, G = oracle.softmax_ce(Zlast, yp, ntrain)
        assert abs(loss - lsum / ntrain) / abs(lsum / ntrain) < 1e-5, (loss, lsum / ntrain)

        # ---- backward, layer by layer from the GPU's Z_G,l
        gm.backward()
        WG = gm.grads()
        ZGs = [mg.mggcn_debug_layer(gm.m, l, (w.n, dims[l + 1])) for l in range(L - 1)]
        inv = oracle.inv_deg(pg.deg_f)
        A_pat = oracle.CSR(pg.A.rowptr, pg.A.col, np.ones(pg.A.col.shape[0], np.float32))   # Â' diag(deg)
        ZG, prescaled = G, False
        for l in range(L - 1, -1, -1):
            J = sorted({0, dims[l + 1] // 2, dims[l + 1] - 1})
            ZJ = np.ascontiguousarray(ZG[:, J])
            A_op = A_pat if prescaled else pg.A
            if order[l] == "G":
                HWG_J = oracle.spmm(A_op, ZJ)                                   # Eq. 9
                ref = oracle.gemm(H[l], HWG_J, transA=True)                     # Eq. 10 (C2)
            else:
                assert l == 0, "SpMM-first layer at l > 0 is not in the configs (C22)"
                T0 = oracle.spmm(pg.At, H[0])                                   # §4.4: T_0 = Â'^T X
                ref = oracle.gemm(T0, ZJ, transA=True)
            assert rel(WG[l][:, J], ref) < REL_TOL, ("W_G", l, rel(WG[l][:, J], ref))
            if l > 0:
                assert order[l] == "G"
                HWG_R = oracle.spmm(A_op, ZG, rows=R)
                ZR = oracle.gemm(HWG_R, Ws[l], transB=True) * (H[l][R] > 0)     # Eq. 11, Eq. 8 mask
                if order[l - 1] == "G":
                    ZR = ZR * inv[R][:, None]                                   # pre-scale (C20)
                assert rel(ZGs[l - 1][R], ZR) < REL_TOL, ("Z_G", l - 1, rel(ZGs[l - 1][R], ZR))
                ZG, prescaled = ZGs[l - 1], order[l - 1] == "G"

        # ---- Adam on the GPU's reduced gradients
        gm.step(lr=0.01)
        Wn = gm.get_weights()
        for l in range(L):
            Wr, m, v = Ws[l].copy(), np.zeros_like(Ws[l]), np.zeros_like(Ws[l])
            oracle.adam(Wr, np.ascontiguousarray(WG[l]), m, v, 1)
            assert np.abs(Wn[l] - Wr).max() <= 1e-6, ("adam", l, np.abs(Wn[l] - Wr).max())
    finally:
        gm.close()
