"""Whole-epoch GPU parity through the C ABI against the CPU oracle:
logits, loss, every W_G, Adam m / v and W after one step (SURVEY.md §8(c)
"GPU-vs-oracle acceptance"; tolerance from BASELINE.json north_star).
Loopback mode runs the P-stage broadcast pipeline with P ranks on one GPU."""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import random_directed

pytestmark = pytest.mark.gpu

REL_TOL = 1e-3


def rel(x, r):
    return float(np.abs(np.asarray(x, np.float64) - r).max() / max(np.abs(r).max(), 1e-30))


@pytest.fixture(scope="module")
def mg():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_balinsc22_b200 as mg
    return mg


def run_library(mg, n, rp, col, vals, X, y, Ws, dims, P, seed, flags, host_inputs=False, steps=1, lr=0.01,
                delay=None, replicas=1, poison=False):
    from paper_conf_icpp_balinsc22_b200 import GCN
    gm = GCN(n, rp, col, vals, dims, P=P, perm_seed=seed, flags=flags, loopback=P > 1, replicas=replicas)
    if delay is not None:                       # (seed, max_us): spin kernels on both streams
        mg.mggcn_debug_comm_delay(gm.m, *delay)
    if poison:                                  # NaN-fill every BC slot right before it is filled
        mg.mggcn_debug_poison(gm.m, int(poison))
    gm.set_weights(Ws)
    Xl = gm.permute_rows(X)
    yl = gm.permute_rows(y)
    if host_inputs:
        Xin, yin = Xl, yl
    else:
        Xin, yin = torch.from_numpy(Xl).cuda(), torch.from_numpy(yl).cuda()
    logits = torch.empty((replicas * n, dims[-1]), dtype=torch.float32, device="cuda")
    out = {}
    for s in range(steps):
        out["loss"] = gm.forward(Xin, yin, want_loss=True, logits=logits if s == 0 else None)
        if s == 0:
            out["logits"] = logits.cpu().numpy()
        gm.backward()
        if s == 0:
            out["WG"] = gm.grads()
        gm.step(lr=lr)
    out["W"] = gm.get_weights()
    out["adam"] = [gm.adam_state(l) for l in range(len(Ws))]
    out["perm"] = gm.perm
    gm.close()
    return out


def compare(lib, ref, dims, tol=REL_TOL):
    assert np.array_equal(lib["perm"], ref.perm)
    assert rel(lib["logits"], ref.logits) < tol, rel(lib["logits"], ref.logits)
    assert abs(lib["loss"] - ref.loss) / abs(ref.loss) < tol, (lib["loss"], ref.loss)
    for l, (a, b) in enumerate(zip(lib["WG"], ref.WG)):
        assert rel(a, b) < tol, (l, rel(a, b))
    for l in range(len(dims) - 1):
        mo, ve, t = lib["adam"][l]
        assert t == 1
        assert rel(mo, ref.m[l]) < tol and rel(ve, ref.v[l]) < tol
        # W where |g| is not tiny, within the first Adam step's own sensitivity (reading C30)
        g, gg = ref.WG[l].astype(np.float64), lib["WG"][l].astype(np.float64)
        mask = np.abs(g) > 1e-3 * np.abs(g).max()
        bound = 1e-5 + 0.01 * np.abs(gg / (np.abs(gg) + 1e-8) - g / (np.abs(g) + 1e-8))
        assert np.all((np.abs(lib["W"][l].astype(np.float64) - ref.W[l]) <= bound)[mask]), l


def workload_inputs(w, unlabelled=0):
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    X = gen.features(w.n, w.dims[0], w.seed_X)
    y = gen.labels(w.n, w.dims[-1], w.seed_y, unlabelled)
    Ws = [gen.glorot(w.dims[l], w.dims[l + 1], w.seed_W + l) for l in range(len(w.dims) - 1)]
    return rp, col, X, y, Ws


@pytest.mark.parametrize("P", [1, 2, 4])
def test_cora_shaped_epoch(mg, P):
    """BASELINE configs[0]: Cora-shaped, 2 layers 1433 -> 16 -> 7."""
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, P, w.perm_seed, mg.MGGCN_F_OVERLAP)
    compare(lib, ref, w.dims)


def test_cora_shaped_unlabelled_host_inputs(mg):
    """10 % unlabelled vertices, inputs given as HOST pointers (the e2e path)."""
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w, unlabelled=100)
    assert (y < 0).sum() > 100
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 1, w.perm_seed, mg.MGGCN_F_OVERLAP,
                      host_inputs=True)
    compare(lib, ref, w.dims)


@pytest.mark.parametrize("P", [1, 3])
@pytest.mark.parametrize("dims", [(8, 32, 32, 5), (100, 256, 256, 47), (24, 16, 12)])
def test_small_rmat_epoch(mg, P, dims):
    """SpMM-first layer 0 (d0 < d1, §4.4) and GeMM-first layers; ragged widths."""
    n, m = 3001, 60000
    rp, col = gen.rmat_csr(n, m, 71)
    X = gen.features(n, dims[0], 72)
    y = gen.labels(n, dims[-1], 73)
    Ws = [gen.glorot(dims[l], dims[l + 1], 74 + l) for l in range(len(dims) - 1)]
    pg = oracle.permute_graph(n, rp, col, None, seed=75)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_library(mg, n, rp, col, None, X, y, Ws, dims, P, 75, mg.MGGCN_F_OVERLAP)
    compare(lib, ref, dims)


@pytest.mark.parametrize("P", [1, 2])
def test_weighted_directed_epoch(mg, P):
    n = 1500
    rp, col, vals = random_directed(n, 20000, 8, weighted=True)
    dims = (20, 16, 6)
    X = gen.features(n, dims[0], 81)
    y = gen.labels(n, dims[-1], 82)
    Ws = [gen.glorot(dims[l], dims[l + 1], 83 + l) for l in range(2)]
    pg = oracle.permute_graph(n, rp, col, vals, seed=84)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_library(mg, n, rp, col, vals, X, y, Ws, dims, P, 84, mg.MGGCN_F_OVERLAP)
    compare(lib, ref, dims)


def test_cora_shaped_no_coalesce(mg):
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 2, w.perm_seed,
                      mg.MGGCN_F_OVERLAP | mg.MGGCN_F_NO_COALESCE)
    compare(lib, ref, w.dims)


@pytest.mark.parametrize("P", [1, 2])
def test_cache_l0_two_epochs(mg, P):
    """MGGCN_F_CACHE_L0: layer 0 runs SpMM-first with T0 = Â'^T X
    computed once; two training steps match the oracle's two steps."""
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    from paper_conf_icpp_balinsc22_b200 import GCN
    gm = GCN(w.n, rp, col, None, w.dims, P=P, perm_seed=w.perm_seed, loopback=P > 1,
             flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_CACHE_L0)
    gm.set_weights(Ws)
    Xd = torch.from_numpy(gm.permute_rows(X)).cuda()
    yd = torch.from_numpy(gm.permute_rows(y)).cuda()
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    Wc, st = [W.copy() for W in Ws], None
    for t in (1, 2):
        ref = oracle.epoch(pg, X, y, Wc, adam_state=st, t=t)
        loss = gm.forward(Xd if t == 1 else Xd * 0, yd)       # 2nd epoch must not read X
        assert abs(loss - ref.loss) / ref.loss < REL_TOL
        gm.backward()
        if t == 1:   # after one Adam step W differs by up to 2 lr where g ~ 0 (sign flips): compare loss only
            for a, b in zip(gm.grads(), ref.WG):
                assert rel(a, b) < REL_TOL
        gm.step()
        Wc, st = ref.W, (ref.m, ref.v)
    gm.close()


def test_relu_last_and_no_overlap(mg):
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    ref = oracle.epoch(pg, X, y, Ws, relu_last=True)
    lib = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 2, w.perm_seed, mg.MGGCN_F_RELU_LAST)
    compare(lib, ref, w.dims)


def test_bitwise_determinism_and_pipeline_invariance(mg):
    """Same inputs twice -> bitwise identical; P-way loopback with and without
    overlap -> bitwise identical (same stage order, only the schedule differs)."""
    n, m = 2000, 40000
    rp, col = gen.rmat_csr(n, m, 91)
    dims = (32, 64, 10)
    X = gen.features(n, dims[0], 92)
    y = gen.labels(n, dims[-1], 93)
    Ws = [gen.glorot(dims[l], dims[l + 1], 94 + l) for l in range(2)]
    a = run_library(mg, n, rp, col, None, X, y, Ws, dims, 3, 95, mg.MGGCN_F_OVERLAP)
    b = run_library(mg, n, rp, col, None, X, y, Ws, dims, 3, 95, mg.MGGCN_F_OVERLAP)
    c = run_library(mg, n, rp, col, None, X, y, Ws, dims, 3, 95, 0)
    for other in (b, c):
        assert np.array_equal(a["logits"], other["logits"])
        assert a["loss"] == other["loss"]
        for x, z in zip(a["WG"], other["WG"]):
            assert np.array_equal(x, z)


def test_multi_step_training_decreases_loss(mg):
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    from paper_conf_icpp_balinsc22_b200 import GCN
    gm = GCN(w.n, rp, col, None, w.dims, perm_seed=w.perm_seed)
    gm.set_weights(Ws)
    Xd = torch.from_numpy(gm.permute_rows(X)).cuda()
    yd = torch.from_numpy(gm.permute_rows(y)).cuda()
    losses = []
    for _ in range(20):
        losses.append(gm.forward(Xd, yd))
        gm.backward()
        gm.step(lr=0.01)
    assert losses[-1] < losses[0]
    # oracle 3 steps agree
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    Wc = [W.copy() for W in Ws]
    st = None
    gm2 = GCN(w.n, rp, col, None, w.dims, perm_seed=w.perm_seed)
    gm2.set_weights(Ws)
    for t in range(1, 4):
        r = oracle.epoch(pg, X, y, Wc, adam_state=st, t=t)
        lo = gm2.forward(Xd, yd)
        assert abs(lo - r.loss) / r.loss < REL_TOL
        gm2.backward()
        gm2.step()
        Wc, st = r.W, (r.m, r.v)
    gm.close()
    gm2.close()


def test_prefetch_matches_direct_inputs(mg):
    """mggcn_prefetch (next epoch's host inputs copied on the copy stream into the
    second input buffer) gives bitwise the same training as passing X each forward."""
    n, m = 3001, 60000
    rp, col = gen.rmat_csr(n, m, 61)
    dims = (602, 32, 7)
    X = gen.features(n, dims[0], 62)
    y = gen.labels(n, dims[-1], 63, 100)
    Ws = [gen.glorot(dims[l], dims[l + 1], 64 + l) for l in range(2)]
    from paper_conf_icpp_balinsc22_b200 import GCN
    runs = []
    for use_prefetch in (False, True):
        gm = GCN(n, rp, col, None, dims, P=2, perm_seed=65, loopback=True)
        gm.set_weights(Ws)
        Xh = torch.from_numpy(gm.permute_rows(X)).pin_memory()
        yh = torch.from_numpy(gm.permute_rows(y)).pin_memory()
        losses = []
        if use_prefetch:
            gm.prefetch(Xh, yh)
        for k in range(4):
            if use_prefetch:
                losses.append(gm.forward(None, None))
                if k < 3:
                    gm.prefetch(Xh, yh)
            else:
                losses.append(gm.forward(Xh, yh))
            gm.backward()
            gm.step()
        runs.append((losses, gm.get_weights()))
        gm.close()
    assert runs[0][0] == runs[1][0]
    for a, b in zip(runs[0][1], runs[1][1]):
        assert np.array_equal(a, b)


def test_device_zero_copy_inputs(mg):
    """A device X in the padded layout (ld = d0 rounded to 8) is read in place:
    bitwise the same epoch as the staged copy."""
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    from paper_conf_icpp_balinsc22_b200 import GCN
    out = []
    for padded in (False, True):
        gm = GCN(w.n, rp, col, None, w.dims, perm_seed=w.perm_seed)
        gm.set_weights(Ws)
        Xl = gm.permute_rows(X)
        Xd = gm.device_inputs(Xl) if padded else torch.from_numpy(Xl).cuda()
        assert (Xd.shape[1] == 1440) == padded
        yd = torch.from_numpy(gm.permute_rows(y)).cuda()
        losses = []
        for _ in range(3):
            losses.append(gm.forward(Xd, yd))
            gm.backward()
            gm.step()
        out.append((losses, gm.get_weights()))
        gm.close()
    assert out[0][0] == out[1][0]
    for a, b in zip(out[0][1], out[1][1]):
        assert np.array_equal(a, b)


def test_state_errors(mg):
    from paper_conf_icpp_balinsc22_b200 import GCN
    rp, col = gen.rmat_csr(200, 2000, 1)
    gm = GCN(200, rp, col, None, (8, 4))
    with pytest.raises(mg.MggcnError) as e:
        gm.backward()
    assert e.value.code == mg.MGGCN_ESTATE
    with pytest.raises(mg.MggcnError) as e:
        gm.step()
    assert e.value.code == mg.MGGCN_ESTATE
    with pytest.raises(mg.MggcnError) as e:
        gm.forward(None, None)                       # no prefetch pending
    assert e.value.code == mg.MGGCN_ESTATE
    gm.close()
    with pytest.raises(mg.MggcnError) as e:
        GCN(200, rp, col, None, (8, 4, 16, 2))      # SpMM-first at l = 1
    assert e.value.code == mg.MGGCN_EUNSUPPORTED


@pytest.mark.parametrize("dims", [(1433, 16, 7), (100, 256, 47)])
def test_padded_host_inputs_with_nan_padding(mg, dims):
    """Host X in the library's padded row layout (one contiguous H2D, mggcn.h) whose
    padding columns hold NaN: padding is never read as data (GEMM tensor maps stop at
    d_0; the SpMM-first T0 padding is ignored), so the epoch still matches the oracle.
    Also through mggcn_prefetch (the e2e path of bench.py)."""
    from paper_conf_icpp_balinsc22_b200 import GCN
    n, m = 2708, 10556
    rp, col = gen.rmat_csr(n, m, 31)
    X = gen.features(n, dims[0], 32)
    y = gen.labels(n, dims[-1], 33)
    Ws = [gen.glorot(dims[l], dims[l + 1], 34 + l) for l in range(len(dims) - 1)]
    pg = oracle.permute_graph(n, rp, col, None, seed=35)
    ref = oracle.epoch(pg, X, y, Ws)
    for P, use_prefetch in ((1, False), (2, True)):
        gm = GCN(n, rp, col, None, dims, P=P, perm_seed=35, flags=mg.MGGCN_F_OVERLAP, loopback=P > 1)
        gm.set_weights(Ws)
        Xl, yl = gm.permute_rows(X), gm.permute_rows(y)
        Xh = np.full((Xl.shape[0], gm.ld0), np.nan, dtype=np.float32)
        Xh[:, :dims[0]] = Xl
        Xh = torch.from_numpy(Xh).pin_memory()
        yh = torch.from_numpy(yl).pin_memory()
        logits = torch.empty((n, dims[-1]), dtype=torch.float32, device="cuda")
        if use_prefetch:
            gm.prefetch(Xh, yh)
            loss = gm.forward(None, None, want_loss=True, logits=logits)
        else:
            loss = gm.forward(Xh, yh, want_loss=True, logits=logits)
        gm.backward()
        lib = {"perm": gm.perm, "logits": logits.cpu().numpy(), "loss": loss, "WG": gm.grads()}
        gm.step()
        lib["W"] = gm.get_weights()
        lib["adam"] = [gm.adam_state(l) for l in range(len(Ws))]
        gm.close()
        assert np.isfinite(lib["logits"]).all()
        compare(lib, ref, dims)


@pytest.mark.parametrize("dims", [(24, 16, 5), (8, 32, 32, 6)])
def test_solo_timing_mode_on_disconnected_halves(mg, dims):
    """SOLO timing mode (MGGCN_F_NO_BCAST, P = 2, nlocal = 1, no NCCL id): one rank of a 2-way run
    alone, every collective skipped.  On a graph made of two disconnected copies of an R-MAT
    graph with the identity permutation, the off-diagonal tiles are empty, so the skipped
    broadcasts and reductions carry nothing and rank r's epoch is exactly the oracle epoch of
    component r (its own |T|, its own W_G).  Without NO_BCAST the same call is EINVAL."""
    from paper_conf_icpp_balinsc22_b200 import GCN
    n0 = 700
    rp0, col0 = gen.rmat_csr(n0, 12000, 31)
    rp = np.concatenate([rp0, rp0[1:] + rp0[-1]]).astype(np.int64)
    col = np.concatenate([col0, col0 + n0]).astype(np.int32)
    n = 2 * n0
    X = gen.features(n, dims[0], 32)
    y = gen.labels(n, dims[-1], 33)
    Ws = [gen.glorot(dims[l], dims[l + 1], 34 + l) for l in range(len(dims) - 1)]
    flags = mg.MGGCN_F_OVERLAP | mg.MGGCN_F_NO_BCAST
    for rank in (0, 1):
        gm = GCN(n, rp, col, None, dims, P=2, rank=rank, perm_seed=0, flags=flags)
        assert gm.rows == n0 and gm.row0 == rank * n0
        gm.set_weights(Ws)
        sl = slice(rank * n0, (rank + 1) * n0)
        logits = torch.empty((n0, dims[-1]), dtype=torch.float32, device="cuda")
        loss = gm.forward(torch.from_numpy(X[sl].copy()).cuda(), torch.from_numpy(y[sl].copy()).cuda(),
                          want_loss=True, logits=logits)
        gm.backward()
        WG = gm.grads()
        gm.step(lr=0.01)
        W1 = gm.get_weights()
        gm.close()
        ref = oracle.epoch(oracle.permute_graph(n0, rp0, col0, None, seed=0), X[sl], y[sl], Ws)
        assert rel(logits.cpu().numpy(), ref.logits) < REL_TOL
        assert abs(loss - ref.loss) / abs(ref.loss) < REL_TOL
        for a, b in zip(WG, ref.WG):
            assert rel(a, b) < REL_TOL
        for l in range(len(Ws)):
            g = ref.WG[l]
            mask = np.abs(g) > 1e-3 * np.abs(g).max()
            np.testing.assert_allclose(W1[l][mask], ref.W[l][mask], rtol=0, atol=1e-5)
    with pytest.raises(mg.MggcnError) as e:
        GCN(n, rp, col, None, dims, P=2, rank=0, perm_seed=0, flags=mg.MGGCN_F_OVERLAP)
    assert e.value.code == mg.MGGCN_EINVAL


@pytest.mark.parametrize("P,replicas", [(3, 1), (4, 1), (4, 2)])
def test_delay_injection_keeps_results_bitwise(mg, P, replicas):
    """SURVEY §4 pipeline-logic test: spin kernels of pseudo-random length (0..200 us) before
    every broadcast (comm stream) and every SpMM stage (compute stream) reshuffle how the
    two streams interleave, and every BC slot is NaN-poisoned right before it is filled; the
    P:929-941 event rule must keep logits, loss, W_G and the updated W bitwise equal to the
    undelayed run, for several seeds, 1D and 1.5D."""
    n, m = 1500, 30000
    rp, col = gen.rmat_csr(n, m, 71)
    dims = (24, 48, 9)
    X = gen.features(n, dims[0], 72)
    y = gen.labels(n, dims[-1], 73)
    Ws = [gen.glorot(dims[l], dims[l + 1], 74 + l) for l in range(2)]
    base = run_library(mg, n, rp, col, None, X, y, Ws, dims, P, 75, mg.MGGCN_F_OVERLAP, steps=2, replicas=replicas)
    for seed in (1, 2, 3):
        d = run_library(mg, n, rp, col, None, X, y, Ws, dims, P, 75, mg.MGGCN_F_OVERLAP, steps=2,
                        delay=(seed, 200), replicas=replicas, poison=True)
        assert np.array_equal(base["logits"], d["logits"])
        assert base["loss"] == d["loss"]
        for a, b in zip(base["WG"], d["WG"]):
            assert np.array_equal(a, b)
        for a, b in zip(base["W"], d["W"]):
            assert np.array_equal(a, b)
    from paper_conf_icpp_balinsc22_b200 import GCN
    gm = GCN(n, rp, col, None, dims, P=1, perm_seed=75)
    with pytest.raises(mg.MggcnError) as e:
        mg.mggcn_debug_comm_delay(gm.m, 0, 20000)
    assert e.value.code == mg.MGGCN_EINVAL
    gm.close()


def _stage_overlaps(tl):
    """Pairs (comm record of block q, SpMM stage record of another block q') of the same SpMM whose
    device intervals intersect.  (In loopback one comm record holds the copies of block q to every
    receiver, so a receiver's stage of that same block may start before the record ends.)"""
    eps = 2e-3   # ms: event timestamp resolution
    comm = [r for r in tl if r["stream"] == 1 and r["cls"] == "bcast" and r["spmm"] >= 0]
    comp = [r for r in tl if r["stream"] == 0 and r["cls"] == "spmm" and r["spmm"] >= 0]
    return [(a, b) for a in comm for b in comp
            if a["spmm"] == b["spmm"] and a["stage"] != b["stage"] and a["t0"] < b["t1"] - eps
            and b["t0"] < a["t1"] - eps]


@pytest.mark.parametrize("P,replicas", [(4, 1), (4, 2)])
def test_overlap_flag_orders_exchange_and_stages(mg, P, replicas):
    """MGGCN_F_OVERLAP semantics (include/mggcn.h; Fig. 8), checked on the
    per-stage timeline rather than on the numbers: without the flag every broadcast starts only
    after the previous SpMM stage finished (no comm interval intersects a stage interval of the
    same SpMM); with it, broadcast k+1 runs while stage k computes.  Delay injection (spins of up
    to 300 us on both streams) makes both orders observable; results stay bitwise equal."""
    from paper_conf_icpp_balinsc22_b200 import GCN
    n, m = 3000, 120000
    rp, col = gen.rmat_csr(n, m, 81)
    dims = (32, 64, 8)
    X = gen.features(n, dims[0], 82)
    y = gen.labels(n, dims[-1], 83)
    Ws = [gen.glorot(dims[l], dims[l + 1], 84 + l) for l in range(2)]
    res = {}
    for overlap in (False, True):
        flags = mg.MGGCN_F_TIMELINE | (mg.MGGCN_F_OVERLAP if overlap else 0)
        gm = GCN(n, rp, col, None, dims, P=P, perm_seed=85, flags=flags, loopback=True, replicas=replicas)
        mg.mggcn_debug_comm_delay(gm.m, 5, 300)
        gm.set_weights(Ws)
        Xd = torch.from_numpy(gm.permute_rows(X)).cuda()
        yd = torch.from_numpy(gm.permute_rows(y)).cuda()
        loss = gm.forward(Xd, yd, want_loss=True)
        gm.backward()
        tl = mg.mggcn_get_timeline(gm.m)
        res[overlap] = (loss, gm.grads(), _stage_overlaps(tl), tl)
        gm.close()
    tl_off = res[False][3]
    assert any(r["stream"] == 1 and r["cls"] == "bcast" for r in tl_off)
    assert any(r["stream"] == 0 and r["cls"] == "spmm" and r["stage"] >= 0 for r in tl_off)
    assert res[False][2] == [], res[False][2][:3]
    assert len(res[True][2]) > 0
    assert res[False][0] == res[True][0]
    for a, b in zip(res[False][1], res[True][1]):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("var,group", [("MGGCN_STAGE_GROUP", "1"), ("MGGCN_STAGE_GROUP", "3"),
                                       ("MGGCN_STAGE_GROUP", "7"), ("MGGCN_STAGE_GROUPS", "3,4"), (None, None)])
def test_stage_group_sizes_epoch(mg, monkeypatch, var, group):
    """Loopback P = 8 epochs with 1 (the paper's one launch per stage), 3, 7 and (3, 4) remote
    blocks per launch and the default grouping match the oracle (logits, loss, W_G, Adam) and
    are bitwise reproducible under delay injection (a group launch waits for the last block of
    its group)."""
    if var:
        monkeypatch.setenv(var, group)
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    ref = oracle.epoch(oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed), X, y, Ws)
    a = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 8, w.perm_seed, mg.MGGCN_F_OVERLAP)
    compare(a, ref, w.dims)
    b = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 8, w.perm_seed, mg.MGGCN_F_OVERLAP, delay=(9, 150),
                    poison=True)
    assert np.array_equal(a["logits"], b["logits"]) and a["loss"] == b["loss"]
    for u, v in zip(a["W"], b["W"]):
        assert np.array_equal(u, v)


@pytest.mark.parametrize("group", ["1", None])
def test_poison_negative_control(mg, monkeypatch, group):
    """The poison check has teeth: with the compute stream's broadcast waits dropped
    (mggcn_debug_poison(m, 2)) and long spins on the comm stream, stages read BC slots that
    were NaN-filled but not yet refilled, so the epoch's logits are no longer the oracle's;
    the same run with the waits kept (poison 1) is bitwise equal to the clean run."""
    if group:
        monkeypatch.setenv("MGGCN_STAGE_GROUP", group)
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    clean = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 4, w.perm_seed, mg.MGGCN_F_OVERLAP)
    good = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 4, w.perm_seed, mg.MGGCN_F_OVERLAP,
                       delay=(3, 2000), poison=1)
    assert np.array_equal(clean["logits"], good["logits"])
    bad = run_library(mg, w.n, rp, col, None, X, y, Ws, w.dims, 4, w.perm_seed, mg.MGGCN_F_OVERLAP,
                      delay=(3, 2000), poison=2)
    assert not np.array_equal(np.nan_to_num(bad["logits"], nan=1e30), clean["logits"])


def test_stage_group_regimes(mg):
    """choose_groups: a rank whose blocks compute longer than they take to arrive
    (many entries per row per tile) gets two groups; an exchange-bound one keeps a last group of
    one block (its tail after the last arrival is one block, as in the per-stage schedule)."""
    from paper_conf_icpp_balinsc22_b200 import GCN
    dims = (16, 16, 4)
    n = 3000
    rp, col = gen.rmat_csr(n, 2000000, 91)           # ~670 entries per row: ~80 per row per tile at P = 8
    gm = GCN(n, rp, col, None, dims, P=8, perm_seed=1, loopback=True)
    assert mg.mggcn_stage_groups(gm.m) == [2, 5]
    gm.close()
    rp, col = gen.rmat_csr(n, 30000, 92)             # ~10 entries per row: ~1 per tile
    gm = GCN(n, rp, col, None, dims, P=8, perm_seed=1, loopback=True)
    assert mg.mggcn_stage_groups(gm.m) == [2, 4, 1]
    gm.close()
    gm = GCN(n, rp, col, None, dims, P=3, perm_seed=1, loopback=True)
    assert mg.mggcn_stage_groups(gm.m) == []         # P <= 3: the paper's per-stage schedule
    gm.close()
