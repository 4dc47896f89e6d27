"""Pins for the shared seeded input generators (gen/).  CPU only."""
import numpy as np
import pytest

import gen


# Random123 known-answer vectors for philox4x32-10 (kat_vectors: ctr, key -> out).
KAT = [
    ((0, 0, 0, 0), (0, 0), (0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8)),
    ((0xFFFFFFFF,) * 4, (0xFFFFFFFF,) * 2, (0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD)),
    ((0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344), (0xA4093822, 0x299F31D0),
     (0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1)),
]


@pytest.mark.parametrize("ctr,key,out", KAT)
def test_philox_kat(ctr, key, out):
    assert tuple(int(x) for x in gen.philox4x32(ctr, key)) == out


def test_uniform_is_24bit_grid():
    u = gen.uniform(7, 0, 10000)
    assert u.min() >= 0 and u.max() < 1
    assert np.all((u * 2 ** 24) == np.floor(u * 2 ** 24))
    # U(seed, i) = word i%4 of Philox(seed, (i/4, 0, 0, 0)) >> 8, 2^-24
    w = gen.philox4x32((1, 0, 0, 0), (7, 0))
    assert u[5] == (int(w[1]) >> 8) / 2 ** 24


@pytest.mark.parametrize("n,m", [(2708, 10556), (1000, 4000), (37, 100)])
def test_rmat_csr_structure(n, m):
    rp, col = gen.rmat_csr(n, m, 1234)
    assert rp[0] == 0 and rp[-1] == m and col.shape == (m,)
    assert col.min() >= 0 and col.max() < n
    rows = np.repeat(np.arange(n), np.diff(rp))
    assert not np.any(rows == col), "no self loops"
    # sorted by (row, col)
    key = rows.astype(np.int64) * n + col
    assert np.all(np.diff(key) >= 0)
    # multiset-symmetric: (u,v) multiplicity == (v,u) multiplicity
    kt = col.astype(np.int64) * n + rows
    assert np.array_equal(np.sort(key), np.sort(kt))
    # deterministic
    rp2, col2 = gen.rmat_csr(n, m, 1234)
    assert np.array_equal(rp, rp2) and np.array_equal(col, col2)


def test_rmat_pairs_follow_recipe():
    """Re-derive the first accepted candidates one by one from Philox words."""
    n = 3000
    s = int(np.ceil(np.log2(n)))
    U, V, used = gen.rmat_pairs(n, 50, 99)
    T1, T2, T3 = 2448131358, 3264175144, 4080218931
    got = []
    k = 0
    while len(got) < 50:
        u = v = 0
        for lvl in range(s):
            if lvl % 4 == 0:
                w = gen.philox4x32((k & 0xFFFFFFFF, k >> 32, lvl // 4, 0), (99, 0))
            r = int(w[lvl % 4])
            bu, bv = (0, 0) if r < T1 else (0, 1) if r < T2 else (1, 0) if r < T3 else (1, 1)
            u, v = 2 * u + bu, 2 * v + bv
        if u < n and v < n and u != v:
            got.append((u, v))
        k += 1
    assert got == list(zip(U.tolist(), V.tolist()))
    assert used == k


def test_rmat_power_law_skew():
    rp, col = gen.rmat_csr(4096, 200000, 5)
    deg = np.diff(rp)
    assert deg.max() > 20 * deg.mean()          # hub rows (load-imbalance stress)
    assert deg[0] == deg.max()                  # natural order puts the hub at id 0


def test_features_labels_weights():
    X = gen.features(100, 13, 42, ld=16)
    assert X.shape == (100, 16) and np.all(X[:, 13:] == 0)
    assert X[:, :13].min() >= -1 and X[:, :13].max() < 1
    u = gen.uniform(42, 0, 13 * 100).reshape(100, 13)
    assert np.array_equal(X[:, :13], (2 * u - 1).astype(np.float32))
    y = gen.labels(1000, 41, 3)
    assert y.min() >= 0 and y.max() < 41
    k24 = (gen.uniform(3, 0, 1000) * 2 ** 24).astype(np.int64)
    assert np.array_equal(y, ((k24 * 41) >> 24).astype(np.int32))
    yu = gen.labels(10000, 7, 3, unlabelled_per_mille=100)
    frac = (yu < 0).mean()
    assert 0.08 < frac < 0.12
    W = gen.glorot(602, 256, 11)
    a = gen.glorot_bound(602, 256)
    assert np.abs(W).max() <= a and np.abs(W).max() > 0.99 * a
