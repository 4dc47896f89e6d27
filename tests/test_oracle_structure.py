"""Oracle pins for the integer / structural part: normalisation (Eq. 2),
permutation (§5.2), partition vector (Eq. 13) and tiles (Eq. 14-15)."""
import numpy as np
import pytest

import oracle
from helpers import csr_from_edges, dense_ahat, fp32_third, golden_val, load_golden, random_directed


def test_normalise_closed_forms():
    # star: k in-edges into vertex 0 -> each Â = 1/k ("average of neighbours" P:963-965)
    k = 7
    rp, col, _ = csr_from_edges(k + 1, [(i, 0) for i in range(1, k + 1)])
    deg, ah = oracle.normalise(k + 1, rp, col)
    assert deg[0] == k and np.all(deg[1:] == 0)
    assert np.all(ah == np.float32(1) / np.float32(k))
    # directed cycle -> every Â = 1
    n = 9
    rp, col, _ = csr_from_edges(n, [(i, (i + 1) % n) for i in range(n)])
    deg, ah = oracle.normalise(n, rp, col)
    assert np.all(deg == 1) and np.all(ah == 1)
    # complete K_n -> 1/(n-1)
    n = 6
    rp, col, _ = csr_from_edges(n, [(i, j) for i in range(n) for j in range(n) if i != j])
    deg, ah = oracle.normalise(n, rp, col)
    assert np.all(ah == np.float32(1) / np.float32(n - 1))


@pytest.mark.parametrize("weighted", [False, True])
def test_normalise_column_stochastic(weighted):
    rp, col, vals = random_directed(50, 400, 3, weighted=weighted)
    deg, ah = oracle.normalise(50, rp, col, vals)
    sums = np.bincount(col, weights=ah.astype(np.float64), minlength=50)
    has_in = deg > 0
    np.testing.assert_allclose(sums[has_in], 1.0, rtol=0, atol=1e-5)
    assert np.all(sums[~has_in] == 0)
    # matches dense brute force
    Ah = dense_ahat(50, rp, col, vals)
    u = np.repeat(np.arange(50), np.diff(rp))
    D = np.zeros((50, 50))
    np.add.at(D, (u, col), ah.astype(np.float64))
    np.testing.assert_allclose(D, Ah, rtol=1e-6, atol=0)


def test_validation_rejects_bad_csr():
    with pytest.raises(ValueError):
        oracle.normalise(3, np.array([0, 1, 1, 3]), np.array([1, 5, 0]))
    with pytest.raises(ValueError):
        oracle.normalise(3, np.array([0, 2, 1, 3]), np.array([1, 2, 0]))
    with pytest.raises(ValueError):
        oracle.normalise(3, np.array([0, 1, 2, 3]), np.array([1, 2, 0]), np.array([1.0, -1.0, 1.0]))


def test_splitmix64_known_values():
    # splitmix64 from state 0 (Steele/Lea/Flood; reference implementation by Vigna)
    assert oracle.splitmix64(0, 3) == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


def test_permutation_properties():
    assert np.array_equal(oracle.permutation(100, 0), np.arange(100))
    for n in (1, 2, 3, 1000):
        p = oracle.permutation(n, 12345)
        assert np.array_equal(np.sort(p), np.arange(n))
    p1, p2 = oracle.permutation(1000, 1), oracle.permutation(1000, 2)
    assert not np.array_equal(p1, p2)
    # Fisher-Yates step by step from the splitmix64 stream (reading C15)
    n, seed = 17, 99
    stream = oracle.splitmix64(seed, n - 1)
    perm = list(range(n))
    for i, k in enumerate(range(n - 1, 0, -1)):
        j = (stream[i] * (k + 1)) >> 64
        perm[k], perm[j] = perm[j], perm[k]
    assert np.array_equal(oracle.permutation(n, seed), perm)


def test_partition_vector():
    assert list(oracle.partition_vector(10, 4)) == [0, 2, 5, 7, 10]
    assert list(oracle.partition_vector(4, 2)) == [0, 2, 4]
    big = oracle.partition_vector(111059956, 8)
    assert big[-1] == 111059956 and np.all(np.diff(big) >= 13882494)


def test_tiles_golden_p2():
    g = load_golden("ka_graph.json")
    pg = oracle.permute_graph(g["n"], np.array(g["rowptr"]), np.array(g["col"], np.int32), None, 0)
    gt = g["tiles_P2"]
    for rank in range(2):
        t = oracle.tiles(pg, 2, rank)
        assert list(t["p"]) == gt["p"]
        for name in ("F", "B"):
            for j in range(2):
                rp, cl, vl = t[name][j]
                grp, gcl, gvl = gt[name][rank][j]
                assert rp.tolist() == grp and cl.tolist() == gcl
                assert [x.view(np.uint32) for x in vl] == [golden_val(x).view(np.uint32) for x in gvl]
        assert [x.view(np.uint32) for x in t["inv_deg"]] == \
            [golden_val(x).view(np.uint32) for x in gt["inv_deg"][rank]]
    assert fp32_third().view(np.uint32) == 0x3EAAAAAB


@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_tiles_roundtrip(P):
    n = 61
    rp, col, vals = random_directed(n, 500, 7, weighted=True)
    pg = oracle.permute_graph(n, rp, col, vals, seed=77)
    Ah = dense_ahat(n, rp, col, vals)
    Pm = oracle.permutation(n, 77)
    Ahp = np.zeros_like(Ah)
    Ahp[np.ix_(Pm, Pm)] = Ah                       # Â'[perm[u], perm[v]] = Â[u, v]
    p = oracle.partition_vector(n, P)
    F = np.zeros((n, n))
    B = np.zeros((n, n))
    total = 0
    for i in range(P):
        t = oracle.tiles(pg, P, i)
        for j in range(P):
            for name, M in (("F", F), ("B", B)):
                trp, tcl, tvl = t[name][j]
                assert trp[0] == 0 and np.all(np.diff(trp) >= 0)
                for r in range(p[i + 1] - p[i]):
                    cols = tcl[trp[r]:trp[r + 1]]
                    assert np.all(np.diff(cols) >= 0), "sorted ascending by local column"
                    assert np.all((cols >= 0) & (cols < p[j + 1] - p[j]))
                    for c, v in zip(cols, tvl[trp[r]:trp[r + 1]]):
                        M[p[i] + r, p[j] + c] += v
                if name == "F":
                    total += trp[-1]
    assert total == rp[-1]
    np.testing.assert_allclose(F, Ahp.T, rtol=1e-6, atol=0)     # F tiles reassemble Â'^T
    np.testing.assert_allclose(B, Ahp, rtol=1e-6, atol=0)       # B tiles reassemble Â'
