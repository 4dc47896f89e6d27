"""Captured epochs (mggcn_epoch_capture / mggcn_epoch_replay): N graph replays
must be BITWISE the same as N eager forward -> backward -> step epochs (same
kernels, same order, Adam's bias corrections re-set per replay), and so carry
the eager path's oracle parity (tests/test_gpu_epoch.py); one replay is also
checked against the CPU oracle directly.  Inputs refilled in place between
replays are read by the next replay.  Error contract of include/mggcn.h."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def mg():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_balinsc22_b200 as mg
    return mg


def make(mg, n, rp, col, dims, P, seed, flags):
    from paper_conf_icpp_balinsc22_b200 import GCN
    return GCN(n, rp, col, None, dims, P=P, perm_seed=seed, flags=flags, loopback=P > 1)


def state(gm, L):
    return gm.get_weights(), [gm.adam_state(l) for l in range(L)], gm.loss()


def small_case(dims):
    n, m = 3001, 60000
    rp, col = gen.rmat_csr(n, m, 91)
    X = gen.features(n, dims[0], 92)
    y = gen.labels(n, dims[-1], 93, 300)
    Ws = [gen.glorot(dims[l], dims[l + 1], 94 + l) for l in range(len(dims) - 1)]
    return n, rp, col, X, y, Ws


@pytest.mark.parametrize("P", [1, 3])
@pytest.mark.parametrize("dims", [(8, 32, 32, 5), (100, 256, 256, 47)])
def test_replay_bitwise_equals_eager(mg, P, dims):
    n, rp, col, X, y, Ws = small_case(dims)
    L = len(dims) - 1
    epochs = 3
    eager = make(mg, n, rp, col, dims, P, 95, mg.MGGCN_F_OVERLAP)
    eager.set_weights(Ws)
    Xd = torch.from_numpy(eager.permute_rows(X)).cuda()
    yd = torch.from_numpy(eager.permute_rows(y)).cuda()
    for _ in range(epochs):
        eager.forward(Xd, yd, want_loss=False)
        eager.backward()
        eager.step(lr=0.01)
    We, Ae, le = state(eager, L)
    eager.close()

    g = make(mg, n, rp, col, dims, P, 95, mg.MGGCN_F_OVERLAP)
    g.set_weights(Ws)
    g.capture_epoch(Xd, yd, lr=0.01)
    # capturing runs nothing: weights and Adam state are untouched
    for l in range(L):
        assert np.array_equal(g.get_weights()[l], Ws[l])
        assert g.adam_state(l)[2] == 0
    g.replay_epoch(1)
    g.replay_epoch(epochs - 1)
    Wg, Ag, lg = state(g, L)
    g.close()
    assert lg == le
    for l in range(L):
        assert np.array_equal(Wg[l], We[l]), l
        for a, b in zip(Ag[l][:2], Ae[l][:2]):
            assert np.array_equal(a, b), l
        assert Ag[l][2] == Ae[l][2] == epochs


def test_replay_matches_oracle_cora(mg):
    """One replayed epoch of BASELINE configs[0] against the CPU oracle (Adam's first
    moment after one step, m = (1 - beta1) W_G, and the loss)."""
    w = gen.WORKLOADS["cora"]
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    X = gen.features(w.n, w.dims[0], w.seed_X)
    y = gen.labels(w.n, w.dims[-1], w.seed_y)
    Ws = [gen.glorot(w.dims[l], w.dims[l + 1], w.seed_W + l) for l in range(len(w.dims) - 1)]
    ref = oracle.epoch(oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed), X, y, Ws)
    g = make(mg, w.n, rp, col, w.dims, 1, w.perm_seed, mg.MGGCN_F_OVERLAP)
    g.set_weights(Ws)
    Xd = torch.from_numpy(g.permute_rows(X)).cuda()
    yd = torch.from_numpy(g.permute_rows(y)).cuda()
    g.capture_epoch(Xd, yd, lr=0.01)
    g.replay_epoch(1)
    loss = g.loss()
    assert abs(loss - ref.loss) / ref.loss < 1e-3
    for l in range(len(Ws)):
        mom, _, t = g.adam_state(l)
        assert t == 1
        np.testing.assert_allclose(mom, ref.m[l], rtol=0, atol=1e-3 * np.abs(ref.m[l]).max())
    g.close()


def test_replay_reads_refilled_inputs(mg):
    """The graph keeps the X/y addresses: new contents written in place are used."""
    dims = (24, 16, 12)
    n, rp, col, X, y, Ws = small_case(dims)
    X2 = gen.features(n, dims[0], 99)
    eager = make(mg, n, rp, col, dims, 1, 96, mg.MGGCN_F_OVERLAP)
    eager.set_weights(Ws)
    for Xi in (X, X2):
        eager.forward(eager.permute_rows(Xi), eager.permute_rows(y), want_loss=False)
        eager.backward()
        eager.step(lr=0.01)
    We, Ae, le = state(eager, 2)
    eager.close()
    g = make(mg, n, rp, col, dims, 1, 96, mg.MGGCN_F_OVERLAP)
    g.set_weights(Ws)
    Xd = torch.from_numpy(g.permute_rows(X)).cuda()
    yd = torch.from_numpy(g.permute_rows(y)).cuda()
    g.capture_epoch(Xd, yd, lr=0.01)
    g.replay_epoch(1)
    g.cs.synchronize()
    with torch.cuda.stream(g.cs):
        Xd.copy_(torch.from_numpy(g.permute_rows(X2)))
    g.replay_epoch(1)
    Wg, Ag, lg = state(g, 2)
    g.close()
    assert lg == le
    for l in range(2):
        assert np.array_equal(Wg[l], We[l])


def test_capture_errors(mg):
    dims = (24, 16, 12)
    n, rp, col, X, y, Ws = small_case(dims)
    g = make(mg, n, rp, col, dims, 1, 97, mg.MGGCN_F_OVERLAP)
    g.set_weights(Ws)
    Xl, yl = g.permute_rows(X), g.permute_rows(y)
    Xd, yd = torch.from_numpy(Xl).cuda(), torch.from_numpy(yl).cuda()
    with pytest.raises(mg.MggcnError) as e:
        mg.mggcn_epoch_replay(g.m, 1)                     # nothing captured
    assert e.value.code == mg.MGGCN_ESTATE
    with pytest.raises(mg.MggcnError) as e:
        mg.mggcn_epoch_capture(g.m, Xl, dims[0], yl)      # host inputs cannot be baked in
    assert e.value.code == mg.MGGCN_EINVAL
    g.forward(Xd, yd, want_loss=False)
    with pytest.raises(mg.MggcnError) as e:
        g.capture_epoch(Xd, yd)                           # mid-epoch
    assert e.value.code == mg.MGGCN_ESTATE
    g.backward()
    g.step()
    g.capture_epoch(Xd, yd)
    with pytest.raises(mg.MggcnError) as e:
        mg.mggcn_epoch_replay(g.m, 0)
    assert e.value.code == mg.MGGCN_EINVAL
    before = mg.mggcn_kernel_launch_count()
    g.replay_epoch(2)
    per = (mg.mggcn_kernel_launch_count() - before) // 2
    assert per > 5
    g.close()
    c = make(mg, n, rp, col, (8, 32, 5), 1, 97, mg.MGGCN_F_OVERLAP | mg.MGGCN_F_CACHE_L0)
    c.set_weights([gen.glorot(8, 32, 1), gen.glorot(32, 5, 2)])
    X8 = torch.from_numpy(c.permute_rows(gen.features(n, 8, 3))).cuda()
    with pytest.raises(mg.MggcnError) as e:
        c.capture_epoch(X8, yd)
    assert e.value.code == mg.MGGCN_EUNSUPPORTED
    c.close()


def test_eager_and_prefetch_after_replay(mg):
    """Replays then eager epochs (prefetched host inputs, the e2e path) = all-eager epochs."""
    dims = (24, 16, 12)
    n, rp, col, X, y, Ws = small_case(dims)

    def run(use_graph):
        g = make(mg, n, rp, col, dims, 1, 98, mg.MGGCN_F_OVERLAP)
        g.set_weights(Ws)
        Xl, yl = g.permute_rows(X), g.permute_rows(y)
        Xd, yd = torch.from_numpy(Xl).cuda(), torch.from_numpy(yl).cuda()
        if use_graph:
            g.capture_epoch(Xd, yd, lr=0.01)
            g.replay_epoch(2)
        else:
            for _ in range(2):
                g.forward(Xd, yd, want_loss=False)
                g.backward()
                g.step(lr=0.01)
        Xh, yh = torch.from_numpy(Xl).pin_memory(), torch.from_numpy(yl).pin_memory()
        g.prefetch(Xh, yh)
        g.forward(None, None, want_loss=False)
        g.backward()
        g.step(lr=0.01)
        out = state(g, 2)
        g.close()
        return out

    We, Ae, le = run(False)
    Wg, Ag, lg = run(True)
    assert lg == le
    for l in range(2):
        assert np.array_equal(Wg[l], We[l])
        assert Ag[l][2] == Ae[l][2] == 3
