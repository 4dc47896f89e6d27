"""C-ABI library: loads, exports every declared symbol, and its host-side
ingest / permutation / partition is BIT-EXACT against the oracle's
independent implementation (CPU only, no GPU needed)."""
import os
import re

import numpy as np
import pytest

import gen
import oracle
from helpers import csr_from_edges, golden_val, load_golden, random_directed

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def mg():
    import build_mggcn
    build_mggcn.build()
    import paper_conf_icpp_balinsc22_b200 as mg
    return mg


def test_exports_every_declared_symbol(mg):
    hdr = open(os.path.join(ROOT, "include", "mggcn.h")).read()
    declared = set(re.findall(r"\b(mggcn_[a-z0-9_]+)\s*\(", hdr))
    assert len(declared) >= 25
    lib = mg.lib()
    for name in sorted(declared):
        assert hasattr(lib, name), f"{name} not exported"
    assert declared == set(mg.EXPORTS)
    assert mg.mggcn_version() >= 100


def test_load_csr_validation(mg):
    with pytest.raises(mg.MggcnError) as e:
        mg.mggcn_load_csr(3, np.array([0, 1, 1, 3]), np.array([1, 5, 0]))
    assert e.value.code == mg.MGGCN_EINVAL
    with pytest.raises(mg.MggcnError):
        mg.mggcn_load_csr(3, np.array([0, 2, 1, 3]), np.array([1, 2, 0]))
    with pytest.raises(mg.MggcnError):
        mg.mggcn_load_csr(3, np.array([0, 1, 2, 3]), np.array([1, 2, 0]), np.array([1.0, 0.0, 1.0]))
    with pytest.raises(mg.MggcnError):
        mg.mggcn_load_csr(0, np.array([0]), np.array([], np.int32))
    g = mg.mggcn_load_csr(3, np.array([0, 1, 2, 3]), np.array([1, 2, 0]))
    with pytest.raises(mg.MggcnError):
        mg.mggcn_partition(g, 4, 0, 0)          # n < P
    with pytest.raises(mg.MggcnError):
        mg.mggcn_partition(g, 2, 2, 0)          # rank out of range
    mg.mggcn_graph_free(g)


@pytest.mark.parametrize("weighted", [False, True])
def test_degree_bitexact(mg, weighted):
    rp, col, vals = random_directed(300, 3000, 4, weighted=weighted)
    g = mg.mggcn_load_csr(300, rp, col, vals)
    info = mg.mggcn_graph_info(g)
    deg, _ = oracle.normalise(300, rp, col, vals)
    assert np.array_equal(info["deg"].view(np.uint32), deg.view(np.uint32))
    assert info["unit_weights"] == (not weighted)
    mg.mggcn_graph_free(g)


def test_symmetry_detection(mg):
    rp, col = gen.rmat_csr(500, 4000, 3)
    g = mg.mggcn_load_csr(500, rp, col)
    assert mg.mggcn_graph_info(g)["symmetric"]
    mg.mggcn_graph_free(g)
    rp, col, _ = random_directed(100, 800, 5)
    g = mg.mggcn_load_csr(100, rp, col)
    assert not mg.mggcn_graph_info(g)["symmetric"]
    mg.mggcn_graph_free(g)


def _compare_part(mg, n, rp, col, vals, P, seed):
    g = mg.mggcn_load_csr(n, rp, col, vals)
    pg = oracle.permute_graph(n, rp, col, vals, seed=seed)
    for rank in range(P):
        part = mg.mggcn_partition(g, P, rank, seed)
        info = mg.mggcn_part_info(part)
        assert np.array_equal(info["perm"], pg.perm)
        t = oracle.tiles(pg, P, rank)
        assert np.array_equal(info["p"], t["p"])
        for d, name in ((0, "F"), (1, "B")):
            for j in range(P):
                lrp, lcol, lval = mg.mggcn_part_export_tile(part, d, j)
                orp, ocol, oval = t[name][j]
                assert np.array_equal(lrp, orp), (rank, name, j)
                assert np.array_equal(lcol, ocol), (rank, name, j)
                assert np.array_equal(lval.view(np.uint32), oval.view(np.uint32)), (rank, name, j)
        assert np.array_equal(mg.mggcn_part_inv_deg(part).view(np.uint32), t["inv_deg"].view(np.uint32))
        mg.mggcn_part_free(part)
    mg.mggcn_graph_free(g)


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_partition_bitexact_rmat(mg, P):
    rp, col = gen.rmat_csr(997, 12000, 77)
    _compare_part(mg, 997, rp, col, None, P, seed=1234 + P)


@pytest.mark.parametrize("P", [1, 2, 5])
@pytest.mark.parametrize("weighted", [False, True])
def test_partition_bitexact_directed(mg, P, weighted):
    rp, col, vals = random_directed(211, 2500, 9, weighted=weighted)
    _compare_part(mg, 211, rp, col, vals, P, seed=0 if P == 5 else 99)


def test_partition_golden_ka(mg):
    g = load_golden("ka_graph.json")
    lg = mg.mggcn_load_csr(g["n"], np.array(g["rowptr"]), np.array(g["col"], np.int32))
    gt = g["tiles_P2"]
    for rank in range(2):
        part = mg.mggcn_partition(lg, 2, rank, 0)
        for d, name in ((0, "F"), (1, "B")):
            for j in range(2):
                rp, cl, vl = mg.mggcn_part_export_tile(part, d, j)
                grp, gcl, gvl = gt[name][rank][j]
                assert rp.tolist() == grp and cl.tolist() == gcl
                assert [v.view(np.uint32) for v in vl] == [golden_val(x).view(np.uint32) for x in gvl]
        mg.mggcn_part_free(part)
    mg.mggcn_graph_free(lg)


def test_partition_cora_shaped_p1(mg):
    w = gen.WORKLOADS["cora"]
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    _compare_part(mg, w.n, rp, col, None, 1, seed=w.perm_seed)


def test_repl2_model_plan_validation(mg):
    """1.5D (MGGCN_F_REPL2) host-side plan checks: loopback needs the
    2P' parts replica-major (part k mod P'), P' must be even, replica 1 is per-process
    only, and the IPC backend is not implemented for it.  The per-rank buffer plan of
    a replicated rank equals that of the 1D rank owning the same row block."""
    n, m = 4096, 60000
    rp, col = gen.rmat_csr(n, m, 5)
    g = mg.mggcn_load_csr(n, rp, col)
    dims = (16, 32, 8)
    R2, R1, IPC = mg.MGGCN_F_REPL2, mg.MGGCN_F_REPLICA1, mg.MGGCN_F_IPC
    try:
        parts2 = [mg.mggcn_partition(g, 2, i, 3) for i in range(2)]
        parts3 = [mg.mggcn_partition(g, 3, i, 3) for i in range(3)]
        b_loop = mg.mggcn_workspace_bytes(parts2 + parts2, dims, R2)
        b_1d = mg.mggcn_workspace_bytes(parts2, dims, 0)
        assert b_loop > b_1d
        one = mg.mggcn_workspace_bytes(parts2[:1], dims, R2)
        assert one == mg.mggcn_workspace_bytes(parts2[:1], dims, R2 | R1) == mg.mggcn_workspace_bytes(parts2[:1], dims, 0)
        bad = [(parts2 + parts2[::-1], R2, mg.MGGCN_EINVAL),       # replica-major order violated
               (parts2, R2, mg.MGGCN_EINVAL),                       # loopback needs 2P' parts
               (parts3 + parts3, R2, mg.MGGCN_EINVAL),              # P' odd
               (parts2[:1], R1, mg.MGGCN_EINVAL),                   # REPLICA1 without REPL2
               (parts2 + parts2, R2 | R1, mg.MGGCN_EINVAL),         # REPLICA1 in loopback
               (parts2[:1], R2 | IPC, mg.MGGCN_EUNSUPPORTED)]
        for parts, flags, code in bad:
            with pytest.raises(mg.MggcnError) as ei:
                mg.mggcn_workspace_bytes(parts, dims, flags)
            assert ei.value.code == code, (flags, ei.value)
        for p in parts2 + parts3:
            mg.mggcn_part_free(p)
    finally:
        mg.mggcn_graph_free(g)
