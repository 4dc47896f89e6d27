"""Oracle pins for the numeric part: SpMM (Eq. 6/9), GEMM (Eq. 5/10/11),
forward (Eq. 5-7, §4.4), softmax-CE, backward (Eq. 8-11),
Adam and the whole epoch.  CPU only; everything is pinned to
something other than the oracle itself (dense brute force, torch autograd,
finite differences, torch.optim.Adam, closed forms, hand-derived values)."""
import math

import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import csr_from_edges, dense_ahat, load_golden, random_directed, torch_epoch


def _ka_graph():
    g = load_golden("ka_graph.json")
    rp, col = np.array(g["rowptr"]), np.array(g["col"], np.int32)
    return g, oracle.permute_graph(g["n"], rp, col, None, 0, dtype=np.float64)


def test_spmm_dense_brute_force():
    n = 40
    rp, col, vals = random_directed(n, 300, 1, weighted=True)
    pg = oracle.permute_graph(n, rp, col, vals, seed=5, dtype=np.float64)
    Ah = dense_ahat(n, rp, col, vals)
    perm = pg.perm
    Ahp = np.zeros_like(Ah)
    Ahp[np.ix_(perm, perm)] = Ah
    B = np.random.default_rng(0).standard_normal((n, 6))
    np.testing.assert_allclose(oracle.spmm(pg.At, B), Ahp.T @ B, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(oracle.spmm(pg.A, B), Ahp @ B, rtol=1e-12, atol=1e-12)
    rows = np.array([3, 0, 39, 17])
    np.testing.assert_array_equal(oracle.spmm(pg.At, B, rows=rows), oracle.spmm(pg.At, B)[rows])


def test_spmm_permutation_graph_is_exact_gather():
    # every in-degree is 1 -> Â^T B is a row gather, bit-exact in fp32
    n = 33
    sigma = np.random.default_rng(2).permutation(n)
    rp, col, _ = csr_from_edges(n, [(u, int(sigma[u])) for u in range(n)])
    pg = oracle.permute_graph(n, rp, col, None, seed=0)
    B = gen.features(n, 5, 9)
    out = oracle.spmm(pg.At, B)
    expect = np.empty_like(B)
    expect[sigma] = B
    assert np.array_equal(out, expect)


@pytest.mark.parametrize("P", [2, 3, 4, 7])
def test_pway_simulation_bit_identical(P):
    rp, col = gen.rmat_csr(500, 6000, 31)
    pg = oracle.permute_graph(500, rp, col, None, seed=3)
    B = gen.features(500, 9, 4)
    p = oracle.partition_vector(500, P)
    one = {"F": oracle.spmm(pg.At, B), "B": oracle.spmm(pg.A, B)}
    blocks = [B[p[j]:p[j + 1]] for j in range(P)]
    for i in range(P):
        t = oracle.tiles(pg, P, i)
        for d in ("F", "B"):
            got = oracle.spmm_tiles(t[d], blocks, 9)
            assert np.array_equal(got, one[d][p[i]:p[i + 1]])


def test_gemm_against_numpy_fp64():
    rng = np.random.default_rng(1)
    A = rng.standard_normal((13, 7))
    B = rng.standard_normal((7, 5))
    np.testing.assert_allclose(oracle.gemm(A, B), A @ B, rtol=1e-13, atol=1e-13)
    np.testing.assert_allclose(oracle.gemm(A, rng.standard_normal((13, 4)), transA=True).shape, (7, 4))
    C = rng.standard_normal((13, 4))
    np.testing.assert_allclose(oracle.gemm(A, C, transA=True), A.T @ C, rtol=1e-13, atol=1e-13)
    D = rng.standard_normal((6, 7))
    np.testing.assert_allclose(oracle.gemm(A, D, transB=True), A @ D.T, rtol=1e-13, atol=1e-13)
    # integer entries: exact in fp32
    Ai = rng.integers(-8, 9, (20, 30)).astype(np.float32)
    Bi = rng.integers(-8, 9, (30, 10)).astype(np.float32)
    assert np.array_equal(oracle.gemm(Ai, Bi), (Ai.astype(np.int64) @ Bi.astype(np.int64)).astype(np.float32))


def test_softmax_ce_closed_form_and_torch():
    C = 7
    Z = np.zeros((5, C))
    y = np.array([0, 3, 6, -1, 2], np.int32)
    s, G = oracle.softmax_ce(Z, y, 4)
    assert abs(s / 4 - math.log(C)) < 1e-14
    for v in (0, 1, 2, 4):
        expect = np.full(C, 1.0 / C)
        expect[y[v]] -= 1.0
        np.testing.assert_allclose(G[v], expect / 4, atol=1e-15)
    assert np.all(G[3] == 0)
    Z = np.random.default_rng(3).standard_normal((50, 11)) * 5
    y = np.random.default_rng(4).integers(-1, 11, 50).astype(np.int32)
    nt = int((y >= 0).sum())
    s, G = oracle.softmax_ce(Z, y, nt)
    Zt = torch.tensor(Z, requires_grad=True)
    yt = torch.tensor(y, dtype=torch.int64)
    lt = torch.nn.functional.cross_entropy(Zt, yt, ignore_index=-1, reduction="mean")
    lt.backward()
    assert abs(s / nt - float(lt)) < 1e-12
    np.testing.assert_allclose(G, Zt.grad.numpy(), atol=1e-14)
    np.testing.assert_allclose(G.sum(axis=1), 0, atol=1e-15)


def test_adam_closed_form_and_torch():
    rng = np.random.default_rng(5)
    W0 = rng.standard_normal(20)
    g = rng.standard_normal(20)
    W, m, v = W0.copy(), np.zeros(20), np.zeros(20)
    oracle.adam(W, g, m, v, 1, lr=0.01)
    np.testing.assert_allclose(W, W0 - 0.01 * g / (np.abs(g) + 1e-8), rtol=0, atol=1e-12)
    # 5 steps vs torch.optim.Adam
    W, m, v = W0.copy(), np.zeros(20), np.zeros(20)
    Wt = torch.tensor(W0.copy(), requires_grad=True)
    opt = torch.optim.Adam([Wt], lr=0.003, betas=(0.9, 0.999), eps=1e-8)
    for t in range(1, 6):
        gt = rng.standard_normal(20)
        oracle.adam(W, gt, m, v, t, lr=0.003)
        Wt.grad = torch.tensor(gt)
        opt.step()
    np.testing.assert_allclose(W, Wt.detach().numpy(), rtol=0, atol=1e-12)


def _random_problem(n, m, dims, seed, weighted=False, unlabelled=0.0):
    rp, col, vals = random_directed(n, m, seed, weighted=weighted)
    rng = np.random.default_rng(seed + 1)
    X = rng.standard_normal((n, dims[0]))
    y = rng.integers(0, dims[-1], n).astype(np.int32)
    if unlabelled:
        y[rng.random(n) < unlabelled] = -1
    Ws = [rng.standard_normal((dims[l], dims[l + 1])) * 0.5 for l in range(len(dims) - 1)]
    return rp, col, vals, X, y, Ws


def _perm_dense(n, rp, col, vals, perm):
    Ah = dense_ahat(n, rp, col, vals)
    Ahp = np.zeros_like(Ah)
    Ahp[np.ix_(perm, perm)] = Ah
    return Ahp


@pytest.mark.parametrize("dims", [(4, 3), (3, 5, 2), (6, 6, 4, 3), (2, 8, 3)])
@pytest.mark.parametrize("relu_last", [False, True])
def test_epoch_vs_torch_autograd(dims, relu_last):
    n = 24
    rp, col, vals, X, y, Ws = _random_problem(n, 120, dims, 11, weighted=True, unlabelled=0.2)
    pg = oracle.permute_graph(n, rp, col, vals, seed=13, dtype=np.float64)
    r = oracle.epoch(pg, X, y, Ws, relu_last=relu_last, dtype=np.float64)
    Xp = np.empty_like(X); Xp[pg.perm] = X
    yp = np.empty_like(y); yp[pg.perm] = y
    logits, loss, grads = torch_epoch(_perm_dense(n, rp, col, vals, pg.perm), Xp, yp, Ws, relu_last)
    np.testing.assert_allclose(r.logits, logits, rtol=1e-10, atol=1e-12)
    assert abs(r.loss - loss) < 1e-12
    for a, b in zip(r.WG, grads):
        np.testing.assert_allclose(a, b, rtol=1e-9, atol=1e-12)


def test_epoch_finite_differences():
    n = 16
    dims = (3, 4, 3)
    rp, col, vals, X, y, Ws = _random_problem(n, 60, dims, 21)
    pg = oracle.permute_graph(n, rp, col, vals, seed=2, dtype=np.float64)
    r = oracle.epoch(pg, X, y, Ws, dtype=np.float64)
    assert min(np.abs(z).min() for z in r.Z[:-1]) > 1e-5      # no ReLU kink within h
    h = 1e-6
    for l in range(len(Ws)):
        for c in range(dims[l]):
            for k in range(dims[l + 1]):
                Wp = [W.copy() for W in Ws]; Wp[l][c, k] += h
                Wm = [W.copy() for W in Ws]; Wm[l][c, k] -= h
                fd = (oracle.epoch(pg, X, y, Wp, dtype=np.float64).loss -
                      oracle.epoch(pg, X, y, Wm, dtype=np.float64).loss) / (2 * h)
                assert abs(fd - r.WG[l][c, k]) <= 1e-6 * max(1.0, abs(fd)), (l, c, k)


def test_forward_dense_brute_force_and_order_swap():
    n = 30
    dims = (5, 9, 4)            # layer 0 S-order (5 < 9), layer 1 G-order
    rp, col, vals, X, y, Ws = _random_problem(n, 150, dims, 31)
    pg = oracle.permute_graph(n, rp, col, vals, seed=8, dtype=np.float64)
    r = oracle.epoch(pg, X, y, Ws, dtype=np.float64)
    assert r.T[0] is not None and r.T[1] is None
    Ahp = _perm_dense(n, rp, col, vals, pg.perm)
    Xp = np.empty_like(X); Xp[pg.perm] = X
    Z0 = Ahp.T @ Xp @ Ws[0]
    Z1 = Ahp.T @ np.maximum(Z0, 0) @ Ws[1]
    np.testing.assert_allclose(r.Z[0], Z0, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(r.logits, Z1, rtol=1e-12, atol=1e-12)
    # associativity of the §4.4 swap: G-order for the same layer agrees to 1e-12
    HW = oracle.gemm(Xp, Ws[0])
    np.testing.assert_allclose(oracle.spmm(pg.At, HW), r.Z[0], rtol=1e-12, atol=1e-12)


def test_permutation_equivariance():
    n = 28
    dims = (4, 6, 3)
    rp, col, vals, X, y, Ws = _random_problem(n, 140, dims, 41)
    pg0 = oracle.permute_graph(n, rp, col, vals, seed=0, dtype=np.float64)
    pg1 = oracle.permute_graph(n, rp, col, vals, seed=999, dtype=np.float64)
    r0 = oracle.epoch(pg0, X, y, Ws, dtype=np.float64)
    r1 = oracle.epoch(pg1, X, y, Ws, dtype=np.float64)
    np.testing.assert_allclose(r1.logits[pg1.perm], r0.logits, rtol=1e-12, atol=1e-12)
    assert abs(r0.loss - r1.loss) < 1e-12
    for a, b in zip(r0.WG, r1.WG):
        np.testing.assert_allclose(a, b, rtol=1e-10, atol=1e-12)


@pytest.mark.parametrize("P", [2, 3, 4])
def test_epoch_pway_matches_1way(P):
    rp, col = gen.rmat_csr(300, 3000, 51)
    X = gen.features(300, 6, 52)
    y = gen.labels(300, 4, 53)
    Ws = [gen.glorot(6, 8, 54), gen.glorot(8, 8, 55), gen.glorot(8, 4, 56)]
    pg = oracle.permute_graph(300, rp, col, None, seed=57)
    r1 = oracle.epoch(pg, X, y, Ws)
    rP = oracle.epoch(pg, X, y, Ws, P=P)
    assert np.array_equal(r1.logits, rP.logits)          # SpMM stages bit-identical
    assert r1.loss == rP.loss
    for a, b in zip(r1.WG, rP.WG):                        # rank-ordered W_G sum: rounding only
        np.testing.assert_allclose(a, b, rtol=1e-5, atol=1e-7)


@pytest.mark.parametrize("case", ["KA1", "KA2"])
def test_known_answers(case):
    g, pg = _ka_graph()
    ka = g[case]
    Ws = [np.array(W, dtype=np.float64) for W in ka["W"]]
    X = np.array(g["X"], dtype=np.float64)
    y = np.array(g["y"], dtype=np.int32)
    r = oracle.epoch(pg, X, y, Ws, dtype=np.float64)
    np.testing.assert_allclose(oracle.spmm(pg.At, X), np.array(g["AtX"]), rtol=0, atol=1e-15)
    np.testing.assert_allclose(r.logits, np.array(ka["logits"]), atol=1e-9)
    assert abs(r.loss - ka["loss"]) < 1e-9
    for a, b in zip(r.WG, ka["WG"]):
        np.testing.assert_allclose(a, np.array(b), atol=1e-9)
    if "Z0" in ka:
        np.testing.assert_allclose(r.Z[0], np.array(ka["Z0"]), atol=1e-9)
    if "W_after_adam_lr0.01" in ka:
        for a, b in zip(r.W, ka["W_after_adam_lr0.01"]):
            np.testing.assert_allclose(a, np.array(b), atol=1e-9)


def test_float_storage_close_to_double():
    rp, col = gen.rmat_csr(400, 4000, 61)
    X = gen.features(400, 12, 62)
    y = gen.labels(400, 5, 63)
    Ws = [gen.glorot(12, 16, 64), gen.glorot(16, 5, 65)]
    pg = oracle.permute_graph(400, rp, col, None, seed=66)
    pg64 = oracle.permute_graph(400, rp, col, None, seed=66, dtype=np.float64)
    r32 = oracle.epoch(pg, X, y, Ws, dtype=np.float32)
    r64 = oracle.epoch(pg64, X, y, Ws, dtype=np.float64)
    rel = np.abs(r32.logits - r64.logits).max() / np.abs(r64.logits).max()
    assert rel < 1e-6
    for a, b in zip(r32.WG, r64.WG):
        assert np.abs(a - b).max() / np.abs(b).max() < 1e-5


@pytest.mark.parametrize("dims", [(3, 5, 2), (6, 6, 4, 3), (2, 8, 3)])
def test_branch_choice_helpers_match_epoch_and_autograd(dims):
    """forward_preactivations / backward_given_masks (reading C31): with the masks Z_l > 0 they
    reproduce oracle.epoch's forward and W_G, and torch float64 autograd (a textbook GCN)."""
    n = 24
    rp, col, vals, X, y, Ws = _random_problem(n, 120, dims, 5, weighted=True, unlabelled=0.2)
    pg = oracle.permute_graph(n, rp, col, vals, seed=7, dtype=np.float64)
    r = oracle.epoch(pg, X, y, Ws, dtype=np.float64)
    Xp = np.empty_like(X); Xp[pg.perm] = X
    yp = np.empty_like(y); yp[pg.perm] = y
    pg32 = oracle.permute_graph(n, rp, col, vals, seed=7)
    Z, H = oracle.forward_preactivations(pg32, Xp, Ws)
    for a, b in zip(Z, r.Z):
        np.testing.assert_allclose(a, b, rtol=1e-5, atol=1e-6)
    ntrain = int((yp >= 0).sum())
    _, G = oracle.softmax_ce(r.logits, yp, ntrain)
    masks = [r.Z[l] > 0 for l in range(len(Ws) - 1)] + [None]
    Hd = [Xp] + [oracle.relu(z) for z in r.Z[:-1]]
    WG = oracle.backward_given_masks(pg, Hd, G, Ws, masks)
    _, _, grads = torch_epoch(_perm_dense(n, rp, col, vals, pg.perm), Xp, yp, Ws)
    for a, b, c in zip(WG, r.WG, grads):
        np.testing.assert_allclose(a, b, rtol=1e-9, atol=1e-12)
        np.testing.assert_allclose(a, c, rtol=1e-9, atol=1e-12)


def test_backward_given_masks_is_the_gradient_of_the_chosen_branch():
    """Flipping one ReLU decision at a pre-activation near 0 changes W_G by exactly the
    gradient of that branch: central finite differences of the loss with the flipped
    mask frozen (the ReLU replaced by the fixed 0/1 mask) match backward_given_masks."""
    n, dims = 16, (3, 4, 3)
    rp, col, vals, X, y, Ws = _random_problem(n, 60, dims, 31)
    pg = oracle.permute_graph(n, rp, col, vals, seed=3, dtype=np.float64)
    Xp = np.empty_like(X); Xp[pg.perm] = X
    yp = np.empty_like(y); yp[pg.perm] = y
    Ahp = _perm_dense(n, rp, col, vals, pg.perm)
    r = oracle.epoch(pg, X, y, Ws, dtype=np.float64)
    mask = r.Z[0] > 0
    i = np.unravel_index(np.argmin(np.abs(r.Z[0])), mask.shape)
    mask[i] = ~mask[i]                                            # the other branch at the smallest |Z|

    def loss_of(Wl):
        H1 = (Ahp.T @ Xp @ Wl[0]) * mask
        Zl = Ahp.T @ H1 @ Wl[1]
        zz = Zl - Zl.max(axis=1, keepdims=True)
        lse = np.log(np.exp(zz).sum(axis=1)) + Zl.max(axis=1)
        lab = yp >= 0
        return float((lse[lab] - Zl[lab, yp[lab]]).sum() / lab.sum())

    H1 = (Ahp.T @ Xp @ Ws[0]) * mask
    logits = Ahp.T @ H1 @ Ws[1]
    _, G = oracle.softmax_ce(logits, yp, int((yp >= 0).sum()))
    WG = oracle.backward_given_masks(pg, [Xp, H1], G, Ws, [mask, None])
    h = 1e-6
    for l in range(2):
        for c in range(dims[l]):
            for k in range(dims[l + 1]):
                Wp = [W.copy() for W in Ws]; Wp[l][c, k] += h
                Wm = [W.copy() for W in Ws]; Wm[l][c, k] -= h
                fd = (loss_of(Wp) - loss_of(Wm)) / (2 * h)
                assert abs(fd - WG[l][c, k]) <= 1e-6 * max(1.0, abs(fd)), (l, c, k)
