"""GPU parity of single ops through the C ABI (tcgen05 GEMM, staged SpMM)
against the CPU oracle, on the same seeded inputs.  Needs a B200."""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import csr_from_edges, random_directed

pytestmark = pytest.mark.gpu

REL_TOL = 1e-3   # BASELINE.json north_star: max relative error 1e-3 (fp32 accumulate)


def rel(x, r):
    return float(np.abs(np.asarray(x, np.float64) - r).max() / max(np.abs(r).max(), 1e-30))


@pytest.fixture(scope="module")
def mg():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_balinsc22_b200 as mg
    return mg


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _pad(a, ld):
    out = np.zeros((a.shape[0], ld), dtype=np.float32)
    out[:, :a.shape[1]] = a
    return out


def _gemm(mg, op, A, B, M, N, K, flags=0):
    lda, ldb = A.shape[1], B.shape[1]
    ldc = (N + 3) // 4 * 4
    C = torch.zeros((M, ldc), dtype=torch.float32, device="cuda")
    dA, dB = _dev(A), _dev(B)
    torch.cuda.synchronize()
    mg.mggcn_debug_gemm(op, M, N, K, dA, lda, dB, ldb, C, ldc, flags, 0)
    return C[:, :N].cpu().numpy()


GEMM_SHAPES = [(128, 16, 32), (1000, 41, 602), (300, 256, 100), (517, 7, 1433), (2048, 112, 8),
               (777, 172, 256), (129, 128, 33), (64, 256, 256), (300, 602, 48), (129, 300, 64), (65, 513, 17)]


@pytest.mark.parametrize("op", [0, 1, 2])
@pytest.mark.parametrize("shape", GEMM_SHAPES)
def test_gemm_integer_exact(mg, op, shape):
    """Integer operands in [-8, 8]: exact in tf32 hi/lo and fp32 sums < 2^24 -> bit-exact."""
    M, N, K = shape
    rng = np.random.default_rng(M * 7 + N * 3 + K + op)
    if op == 0:
        A = rng.integers(-8, 9, (M, K)).astype(np.float32)
        B = rng.integers(-8, 9, (K, N)).astype(np.float32)
        ref = oracle.gemm(A, B)
        A, B = _pad(A, (K + 3) // 4 * 4), _pad(B, (N + 3) // 4 * 4)
    elif op == 1:
        A = rng.integers(-8, 9, (M, K)).astype(np.float32)
        B = rng.integers(-8, 9, (N, K)).astype(np.float32)
        ref = oracle.gemm(A, B, transB=True)
        A, B = _pad(A, (K + 3) // 4 * 4), _pad(B, (K + 3) // 4 * 4)
    else:
        A = rng.integers(-8, 9, (K, M)).astype(np.float32)
        B = rng.integers(-8, 9, (K, N)).astype(np.float32)
        ref = oracle.gemm(A, B, transA=True)
        A, B = _pad(A, (M + 3) // 4 * 4), _pad(B, (N + 3) // 4 * 4)
    got = _gemm(mg, op, A, B, M, N, K)
    assert np.array_equal(got, ref), f"max abs diff {np.abs(got - ref).max()}"


@pytest.mark.parametrize("op", [0, 1, 2])
@pytest.mark.parametrize("x1", [False, True])
def test_gemm_random_fp32(mg, op, x1):
    M, N, K = 3001, 256, 602
    rng = np.random.default_rng(11 + op)
    if op == 0:
        A, B = rng.standard_normal((M, K)).astype(np.float32), rng.standard_normal((K, N)).astype(np.float32)
        ref = oracle.gemm(A.astype(np.float64), B.astype(np.float64))
    elif op == 1:
        A, B = rng.standard_normal((M, K)).astype(np.float32), rng.standard_normal((N, K)).astype(np.float32)
        ref = oracle.gemm(A.astype(np.float64), B.astype(np.float64), transB=True)
    else:
        M, K = 602, 20000
        A, B = rng.standard_normal((K, M)).astype(np.float32), rng.standard_normal((K, N)).astype(np.float32)
        ref = oracle.gemm(A.astype(np.float64), B.astype(np.float64), transA=True)
    r4 = lambda a: _pad(a, (a.shape[1] + 3) // 4 * 4)
    got = _gemm(mg, op, r4(A), r4(B), M, N, K, flags=mg.MGGCN_F_TF32X1 if x1 else 0)
    r = rel(got, ref)
    assert r < (2e-3 if x1 else 1e-5), r


def _model(mg, n, rp, col, vals, dims, P, seed, flags=None):
    from paper_conf_icpp_balinsc22_b200 import GCN
    flags = mg.MGGCN_F_OVERLAP if flags is None else flags
    return GCN(n, rp, col, vals, dims, P=P, perm_seed=seed, flags=flags, loopback=P > 1)


def _spmm_check(mg, n, rp, col, vals, P, width, seed, exact, flags=None):
    dims = (max(width, 1), max(width, 1))       # one G-order layer; bc width covers `width`
    gm = _model(mg, n, rp, col, vals, dims, P, seed, flags)
    pg = oracle.permute_graph(n, rp, col, vals, seed=seed)
    ld = (width + 3) // 4 * 4
    rng = np.random.default_rng(width + P)
    if exact:
        Bm = rng.integers(-64, 65, (n, width)).astype(np.float32)
    else:
        Bm = rng.standard_normal((n, width)).astype(np.float32)
    dB = _dev(_pad(Bm, ld))
    out = torch.zeros((n, ld), dtype=torch.float32, device="cuda")
    for d, csr in ((0, pg.At), (1, pg.A)):
        torch.cuda.synchronize()
        mg.mggcn_debug_spmm(gm.m, d, dB, ld, width, out, ld)
        got = out[:, :width].cpu().numpy()
        ref = oracle.spmm(csr, Bm)
        if exact:
            assert np.array_equal(got, ref), (d, np.abs(got - ref).max())
        else:
            refd = oracle.spmm(oracle.CSR(csr.rowptr, csr.col, csr.val.astype(np.float64)), Bm.astype(np.float64))
            assert rel(got, refd) < 1e-5, (d, rel(got, refd))
    gm.close()


def _circulant(n, k):
    """In-neighbours of v: v+1 .. v+2^k (mod n) -> every in/out degree is 2^k."""
    edges = [((v + i) % n, v) for v in range(n) for i in range(1, 2 ** k + 1)]
    return csr_from_edges(n, edges)


@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("width", [4, 7, 16, 41, 100, 256])
def test_spmm_exactness_graph(mg, P, width):
    n = 1037
    rp, col, _ = _circulant(n, 3)
    _spmm_check(mg, n, rp, col, None, P, width, seed=5, exact=True)


@pytest.mark.parametrize("P,group", [(4, None), (5, "1"), (5, "3"), (8, None), (8, "2"), (8, "7")])
def test_spmm_stage_groups_exact(mg, monkeypatch, P, group):
    """Stage groups (model.cu choose_group_size: several remote blocks consumed by one launch
    over a merged tile whose columns address consecutive BC slots): bit-exact on the
    exactness graph for the default grouping and forced group sizes (1 = one launch per
    stage), and within 1e-5 on R-MAT hubs (split rows + fix-up over merged rows)."""
    if group is not None:
        monkeypatch.setenv("MGGCN_STAGE_GROUP", group)
    n = 1037
    rp, col, _ = _circulant(n, 3)
    for width in (7, 48, 256):
        _spmm_check(mg, n, rp, col, None, P, width, seed=5, exact=True)
    n, m = 4096, 400000
    rp, col = gen.rmat_csr(n, m, 17)
    for width in (44, 256):
        _spmm_check(mg, n, rp, col, None, P, width, seed=9, exact=False)


@pytest.mark.parametrize("P", [1, 2, 4])
@pytest.mark.parametrize("width", [8, 44, 48, 100, 128, 172, 256, 512, 600])
@pytest.mark.parametrize("coalesce", [True, False])
def test_spmm_rmat_hubs(mg, P, width, coalesce):
    """R-MAT with hub rows longer than the 2048-entry split (segments + fix-up),
    duplicate entries merged (default) or kept as separate gathers."""
    n, m = 4096, 400000
    rp, col = gen.rmat_csr(n, m, 17)
    assert np.diff(rp).max() > 4 * 2048
    flags = mg.MGGCN_F_OVERLAP | (0 if coalesce else mg.MGGCN_F_NO_COALESCE)
    _spmm_check(mg, n, rp, col, None, P, width, seed=9, exact=False, flags=flags)


@pytest.mark.parametrize("P", [1, 3])
def test_spmm_weighted_directed(mg, P):
    rp, col, vals = random_directed(2000, 30000, 3, weighted=True)
    _spmm_check(mg, 2000, rp, col, vals, P, 64, seed=2, exact=False)


def test_spmm_power_law_exact_hub(mg):
    """A star whose hub has 9000 in-edges (power of two denominators not needed:
    integer features and a pattern sum) checked against the integer sum."""
    n = 9001
    edges = [(u, 0) for u in range(1, n)] + [(0, u) for u in range(1, 50)]
    rp, col, _ = csr_from_edges(n, edges)
    gm = _model(mg, n, rp, col, None, (8, 8), 1, 0)
    B = np.random.default_rng(0).integers(-3, 4, (n, 8)).astype(np.float32)
    out = torch.zeros((n, 8), dtype=torch.float32, device="cuda")
    mg.mggcn_debug_spmm(gm.m, 0, _dev(B), 8, 8, out, 8)
    got = out.cpu().numpy()
    expect0 = B[1:].astype(np.float64).sum(axis=0) / 9000.0
    np.testing.assert_allclose(got[0], expect0, rtol=1e-6, atol=1e-7)
    gm.close()


@pytest.mark.parametrize("win", [64, 128])
def test_spmm_column_windows(win):
    """The windowed gather (launch_spmm splits the width into column windows,
    automatic for L2-sized blocks) against the oracle: re-runs the R-MAT hub
    cases in a fresh process with the window forced to `win` floats."""
    import os
    import subprocess
    import sys
    if os.environ.get("MGGCN_SPMM_WIN"):
        pytest.skip("already inside a forced-window run")
    here = os.path.dirname(os.path.abspath(__file__))
    env = dict(os.environ, MGGCN_SPMM_WIN=str(win))
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", os.path.join(here, "test_gpu_kernels.py"),
                        "-k", "rmat_hubs and (172 or 256 or 512 or 600) and True"], env=env, cwd=os.path.dirname(here),
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout


@pytest.mark.parametrize("hot_mb", ["0", "0.25", "64"])
def test_spmm_hot_classes(hot_mb):
    """L2 priority classes (column indices carry the reuse-rank class in bits 24..31,
    rows of the hottest classes gathered evict_last): forced on for every tile
    (MGGCN_SPMM_HOTCLS=2) with an evict_last budget of none, a few hub rows, or all
    rows, the R-MAT hub and integer-exact cases match the oracle in a fresh process."""
    import os
    import subprocess
    import sys
    if os.environ.get("MGGCN_SPMM_HOTCLS"):
        pytest.skip("already inside a forced-class run")
    here = os.path.dirname(os.path.abspath(__file__))
    env = dict(os.environ, MGGCN_SPMM_HOTCLS="2", MGGCN_SPMM_HOT_MB=hot_mb)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", os.path.join(here, "test_gpu_kernels.py"),
                        "-k", "rmat_hubs or exactness_graph or weighted_directed or power_law"], env=env,
                       cwd=os.path.dirname(here), capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout


def test_gemm_cta_pair_variant():
    """The opt-in CTA-pair row GEMM (MGGCN_ROW_PAIR=1: cluster of 2, tcgen05.mma.cta_group::2,
    each CTA stages half of B) passes the same integer-exact and random GEMM cases in a
    fresh process (shapes with >= 2 M tiles and BN >= 128 take the pair path)."""
    import os
    import subprocess
    import sys
    if os.environ.get("MGGCN_ROW_PAIR"):
        pytest.skip("already inside a forced-variant run")
    here = os.path.dirname(os.path.abspath(__file__))
    env = dict(os.environ, MGGCN_ROW_PAIR="1")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", os.path.join(here, "test_gpu_kernels.py"),
                        "-k", "gemm_integer_exact or gemm_random"], env=env, cwd=os.path.dirname(here),
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout
