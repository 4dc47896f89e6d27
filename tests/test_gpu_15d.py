"""1.5D partitioning with replication factor c = 2 (SURVEY NEXT-4, P:1033-1066;
MGGCN_F_REPL2) on one GPU in LOOPBACK mode (all 2P' ranks in one model):
whole-epoch parity with the CPU oracle (same tolerance as the 1D path), the
two replicas of every row block bitwise equal, and the per-epoch broadcast
volume of the work model against the paper's 1.5D count."""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import random_directed
from test_gpu_epoch import REL_TOL, compare, rel, workload_inputs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def mg():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_balinsc22_b200 as mg
    return mg


def run_15d(mg, n, rp, col, vals, X, y, Ws, dims, P, seed, flags, steps=1, host_inputs=False):
    from paper_conf_icpp_balinsc22_b200 import GCN
    gm = GCN(n, rp, col, vals, dims, P=P, perm_seed=seed, flags=flags, loopback=True, replicas=2)
    gm.set_weights(Ws)
    Xl, yl = gm.permute_rows(X), gm.permute_rows(y)
    assert Xl.shape[0] == 2 * n
    Xin, yin = (Xl, yl) if host_inputs else (torch.from_numpy(Xl).cuda(), torch.from_numpy(yl).cuda())
    logits = torch.empty((2 * n, dims[-1]), dtype=torch.float32, device="cuda")
    out = {"losses": []}
    for s in range(steps):
        loss = gm.forward(Xin, yin, want_loss=True, logits=logits if s == 0 else None)
        out["losses"].append(loss)
        if s == 0:
            lg = logits.cpu().numpy()
            out["logits"], out["logits_r1"] = lg[:n], lg[n:]
            out["loss"] = loss
        gm.backward()
        if s == 0:
            out["WG"] = gm.grads()
        gm.step()
    out["W"] = gm.get_weights()
    out["adam"] = [gm.adam_state(l) for l in range(len(Ws))]
    out["perm"] = gm.perm
    out["work"] = gm.epoch_work()
    gm.close()
    return out


@pytest.mark.parametrize("P", [4, 8])
def test_15d_cora_shaped_epoch(mg, P):
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_15d(mg, w.n, rp, col, None, X, y, Ws, w.dims, P, w.perm_seed, mg.MGGCN_F_OVERLAP)
    assert np.array_equal(lib["logits"], lib["logits_r1"])      # replicas agree bitwise
    compare(lib, ref, w.dims)


@pytest.mark.parametrize("P", [4, 8])
@pytest.mark.parametrize("dims", [(8, 32, 32, 5), (100, 256, 256, 47), (24, 16, 12)])
def test_15d_small_rmat_epoch(mg, P, dims):
    """SpMM-first layer 0 (d0 < d1) and GeMM-first layers, hub rows, ragged widths."""
    n, m = 3001, 60000
    rp, col = gen.rmat_csr(n, m, 71)
    X = gen.features(n, dims[0], 72)
    y = gen.labels(n, dims[-1], 73, 300)
    Ws = [gen.glorot(dims[l], dims[l + 1], 74 + l) for l in range(len(dims) - 1)]
    pg = oracle.permute_graph(n, rp, col, None, seed=75)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_15d(mg, n, rp, col, None, X, y, Ws, dims, P, 75, mg.MGGCN_F_OVERLAP)
    assert np.array_equal(lib["logits"], lib["logits_r1"])
    compare(lib, ref, dims)


def test_15d_weighted_directed_host_inputs_no_overlap(mg):
    n = 1500
    rp, col, vals = random_directed(n, 20000, 8, weighted=True)
    dims = (20, 16, 6)
    X = gen.features(n, dims[0], 81)
    y = gen.labels(n, dims[-1], 82)
    Ws = [gen.glorot(dims[l], dims[l + 1], 83 + l) for l in range(2)]
    pg = oracle.permute_graph(n, rp, col, vals, seed=84)
    ref = oracle.epoch(pg, X, y, Ws)
    lib = run_15d(mg, n, rp, col, vals, X, y, Ws, dims, 4, 84, 0, host_inputs=True)
    assert np.array_equal(lib["logits"], lib["logits_r1"])
    compare(lib, ref, dims)


def test_15d_training_follows_oracle(mg):
    """Three Adam steps: the loss of every step matches the oracle's trajectory."""
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    lib = run_15d(mg, w.n, rp, col, None, X, y, Ws, w.dims, 4, w.perm_seed, mg.MGGCN_F_OVERLAP, steps=3)
    Wc, st = [W.copy() for W in Ws], None
    for t in range(1, 4):
        ref = oracle.epoch(pg, X, y, Wc, adam_state=st, t=t)
        assert abs(lib["losses"][t - 1] - ref.loss) / ref.loss < REL_TOL, (t, lib["losses"][t - 1], ref.loss)
        Wc, st = ref.W, (ref.m, ref.v)


def test_15d_broadcast_volume(mg):
    """Work model: with c = 2 the job receives (P'-1) n sum(d) floats per epoch over all
    ranks (each rank: the blocks of its replica group), against (P-1) n sum(d) for 1D at
    the same P -- the paper's 1.5D saving before the pair all-reduce."""
    w = gen.WORKLOADS["cora"]
    rp, col, X, y, Ws = workload_inputs(w)
    from paper_conf_icpp_balinsc22_b200 import GCN
    for P in (4, 8):
        g15 = GCN(w.n, rp, col, None, w.dims, P=P, perm_seed=w.perm_seed, loopback=True, replicas=2)
        g1 = GCN(w.n, rp, col, None, w.dims, P=P, perm_seed=w.perm_seed, loopback=True)
        gb = GCN(w.n, rp, col, None, w.dims, P=P // 2, perm_seed=w.perm_seed, loopback=True)
        b15, b1 = g15.epoch_work()["bcast_bytes"], g1.epoch_work()["bcast_bytes"]
        # GEMM work: only the root replica of a block multiplies -> the 1D work at P' row blocks
        assert g15.epoch_work()["gemm_flops"] == gb.epoch_work()["gemm_flops"]
        for gm in (g15, g1, gb):
            gm.close()
        Pb = P // 2
        assert abs(b15 / b1 - (Pb - 1) / (P - 1)) < 1e-9, (P, b15, b1)
