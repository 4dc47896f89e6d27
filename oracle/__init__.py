"""CPU oracle for MG-GCN's full-batch GCN epoch — TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with the
CUDA path (``paper_conf_icpp_balinsc22_b200``) and never imports it.

It computes the PLAIN DEFINITION of one unpartitioned full-batch GCN epoch on
the randomly permuted graph: everything MG-GCN does
(partitioning P:637-720, permutation P:1075-1090, overlap P:903-941, order
swap P:943-951, buffer re-use P:827-901) is an exact re-organisation of it.
Structure (validation, normalisation, permutation application, transposition,
tiles) is numpy; the numeric kernels are the single-threaded C++ in
oracle/oracle.cpp (fp64 accumulation, ascending order, one rounding to the
storage dtype).  PAPER.md is cited as P:line.

Pins (tests/test_oracle_*.py, all ``-m "not gpu"``):
  normalise      closed forms (star 1/k, cycle 1, K_n 1/(n-1)), column sums = 1
  permutation    splitmix64 known value, bijection, seed 0 = identity,
                 equivariance of logits / invariance of loss and W_G
  tiles          hand-derived P = 2 golden (tests/golden/ka_tiles_p2.json),
                 round-trip reassembly of Â', nnz conservation
  spmm / gemm    dense fp64 brute force; permutation-matrix graph = row gather
                 (bit-exact); P-way simulation == 1-way (bit-exact)
  forward        dense brute force Z = Â^T H W; S-order == G-order (fp64)
  softmax-CE     uniform logits -> ln C; torch.nn.functional.cross_entropy
  backward       central finite differences (fp64); torch float64 autograd
                 with a dense Â (independent textbook implementation)
  adam           closed-form first step; torch.optim.Adam for 5 steps
  whole epoch    hand-derived known answers KA1 / KA2 (tests/golden/)
  branch choices forward_preactivations / backward_given_masks == epoch and torch
                 autograd with the masks Z > 0; with a flipped mask, == central
                 finite differences of the loss with that mask frozen (reading C31)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle's C++ core (-O2 -ffp-contract=off, single thread)."""
    src = os.path.join(_HERE, "oracle.cpp")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["g++", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-std=c++17",
                               src, "-o", _SO])
    return _SO


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        i64, i32, u64, dbl = ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_double
        lib.orc_permutation.argtypes = [i64, u64, P]
        lib.orc_splitmix64_next.argtypes = [P]
        lib.orc_csr_order.argtypes = [i64, i64, P, P, P, P]
        lib.orc_splitmix64_next.restype = u64
        for s in ("f32", "f64"):
            getattr(lib, f"orc_spmm_{s}").argtypes = [i64, P, P, P, P, i64, i64, P, i64]
            getattr(lib, f"orc_spmm_tiles_{s}").argtypes = [i64, i32, P, P, P, P, i64, i64, P, i64]
            getattr(lib, f"orc_gemm_{s}").argtypes = [i64, i64, i64, P, i64, ctypes.c_int, P, i64,
                                                      ctypes.c_int, P, i64]
            getattr(lib, f"orc_softmax_ce_{s}").argtypes = [i64, i64, P, i64, P, i64, P, i64, P]
            getattr(lib, f"orc_adam_{s}").argtypes = [i64, P, P, P, P, i64, dbl, dbl, dbl, dbl]
        _lib = lib
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def _suf(dtype):
    return "f64" if np.dtype(dtype) == np.float64 else "f32"


# ------------------------------------------------------------------ RNG
def splitmix64(state: int, count: int) -> list:
    """First `count` outputs of splitmix64 from `state` (reading C15)."""
    s = ctypes.c_uint64(state)
    return [_L().orc_splitmix64_next(ctypes.byref(s)) for _ in range(count)]


def permutation(n: int, seed: int) -> np.ndarray:
    """perm[old] = new (§5.2; RNG reading C15)."""
    perm = np.empty(n, dtype=np.int64)
    _L().orc_permutation(n, seed, _p(perm))
    return perm


# ------------------------------------------------------------ graph / Â
@dataclass
class CSR:
    rowptr: np.ndarray   # int64[nrows+1]
    col: np.ndarray      # int64[nnz]
    val: np.ndarray      # float[nnz]


def validate(n, rowptr, col, vals):
    """O1: A in R^{n x n} given as CSR; duplicates are multiplicities."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    col = np.asarray(col)
    if n <= 0 or rowptr.shape != (n + 1,) or rowptr[0] != 0 or np.any(np.diff(rowptr) < 0):
        raise ValueError("bad rowptr")
    if rowptr[-1] != col.shape[0]:
        raise ValueError("rowptr[n] != nnz")
    if col.size and (col.min() < 0 or col.max() >= n):
        raise ValueError("colidx out of range")
    if vals is not None:
        vals = np.asarray(vals, dtype=np.float32)
        if vals.shape != col.shape or not np.all(np.isfinite(vals)) or np.any(vals <= 0):
            raise ValueError("vals must be finite and > 0")


def normalise(n, rowptr, col, vals=None, dtype=np.float32):
    """Eq. 2, reading C1/C18: deg(v) = sum over entries (u,v) of
    A_uv, summed in fp64 in CSR order and rounded to the storage dtype;
    Â_uv = A_uv / deg(v) as one IEEE division in the storage dtype (fp32 for
    the parity reference, fp64 for the self-tests).  Returns (deg, ahat)."""
    validate(n, rowptr, col, vals)
    col = np.asarray(col, dtype=np.int64)
    a = np.ones(col.shape[0], dtype=dtype) if vals is None else np.asarray(vals, dtype=np.float32).astype(dtype)
    deg = np.bincount(col, weights=a.astype(np.float64), minlength=n)   # sequential, CSR order
    deg_f = deg.astype(dtype)
    ahat = (a / deg_f[col]).astype(dtype) if col.size else np.zeros(0, dtype)
    return deg_f, ahat


@dataclass
class PermutedGraph:
    """Â' = Π Â Π^T as two CSRs (P:306-371 use Â^T forward and Â backward)."""
    n: int
    perm: np.ndarray
    deg_f: np.ndarray          # in NEW vertex ids
    At: CSR                    # rows v' (destination), entries u' (in-neighbours)
    A: CSR                     # rows u', entries v' (out-neighbours)
    orig_pos_At: np.ndarray = field(repr=False, default=None)
    orig_pos_A: np.ndarray = field(repr=False, default=None)


def _csr_from_triplets(n, rows, cols, tie, vals):
    """Sort by (row, col, tie) and build a CSR.  `tie` must be ascending in
    input order (the original CSR position, O4's tie rule), so a stable sort
    by (row, col) is that order (orc_csr_order: stable bucket sort by row, then
    a stable sort of each row by column)."""
    assert tie.shape[0] < 2 or np.all(np.diff(tie) > 0)
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    cols = np.ascontiguousarray(cols, dtype=np.int64)
    rowptr = np.empty(n + 1, dtype=np.int64)
    order = np.empty(rows.shape[0], dtype=np.int64)
    _L().orc_csr_order(n, rows.shape[0], _p(rows), _p(cols), _p(rowptr), _p(order))
    return CSR(rowptr, cols[order], vals[order]), order


def permute_graph(n, rowptr, col, vals=None, seed=0, dtype=np.float32) -> PermutedGraph:
    """O2 + O3: normalise on the original CSR, then relabel u -> perm[u]."""
    deg_f, ahat = normalise(n, rowptr, col, vals, dtype)
    perm = permutation(n, seed)
    rowptr = np.asarray(rowptr, dtype=np.int64)
    u = np.repeat(np.arange(n, dtype=np.int64), np.diff(rowptr))
    v = np.asarray(col, dtype=np.int64)
    pos = np.arange(v.shape[0], dtype=np.int64)           # original CSR position (tie rule)
    pu, pv = perm[u], perm[v]
    At, oAt = _csr_from_triplets(n, pv, pu, pos, ahat)
    A, oA = _csr_from_triplets(n, pu, pv, pos, ahat)
    deg_new = np.empty(n, dtype=deg_f.dtype)
    deg_new[perm] = deg_f
    return PermutedGraph(n, perm, deg_new, At, A, pos[oAt], pos[oA])


def partition_vector(n: int, P: int) -> np.ndarray:
    """Eq. 13, uniform reading C14: p(i) = floor(i n / P)."""
    return np.array([(i * n) // P for i in range(P + 1)], dtype=np.int64)


def inv_deg(deg_f):
    """1/deg in fp32, 0 where deg = 0 (reading C20)."""
    out = np.zeros_like(deg_f, dtype=np.float32)
    nz = deg_f != 0
    out[nz] = (np.float32(1.0) / deg_f[nz]).astype(np.float32)
    return out


def tiles(pg: PermutedGraph, P: int, rank: int):
    """Eq. 14-15 with the 1D row distribution of P:705-720:
    rank i owns rows p(i)..p(i+1)-1 of Â'^T (forward tiles F_ij) and of Â'
    (backward tiles B_ij), each split into P column tiles with local column
    indices.  Returns dict(p, F=[(rowptr i32, col i32, val f32)], B=[...], inv_deg)."""
    p = partition_vector(pg.n, P)
    lo, hi = p[rank], p[rank + 1]
    out = {"p": p}
    for name, csr in (("F", pg.At), ("B", pg.A)):
        s, e = csr.rowptr[lo], csr.rowptr[hi]
        rloc = np.repeat(np.arange(hi - lo, dtype=np.int64), np.diff(csr.rowptr[lo:hi + 1]))
        c, v = csr.col[s:e], csr.val[s:e]
        tl = []
        for j in range(P):
            m = (c >= p[j]) & (c < p[j + 1])            # keeps the (col, tie) order of each row
            rp = np.zeros(hi - lo + 1, dtype=np.int32)
            rp[1:] = np.cumsum(np.bincount(rloc[m], minlength=hi - lo))
            tl.append((rp, (c[m] - p[j]).astype(np.int32), v[m].astype(np.float32)))
        out[name] = tl
    out["inv_deg"] = inv_deg(pg.deg_f[lo:hi])
    return out


# -------------------------------------------------------------- numerics
def spmm(csr: CSR, B: np.ndarray, rows=None) -> np.ndarray:
    """out = M·B for a CSR M (Eq. 6 with M = Â'^T, Eq. 9 with M = Â'); fp64 acc.
    `rows` (optional int array) computes only those output rows."""
    dt = B.dtype
    width = B.shape[1]
    Bc = np.ascontiguousarray(B)
    val = np.ascontiguousarray(csr.val.astype(dt))
    if rows is None:
        nrows = csr.rowptr.shape[0] - 1
        out = np.empty((nrows, width), dtype=dt)
        getattr(_L(), f"orc_spmm_{_suf(dt)}")(nrows, _p(csr.rowptr), _p(csr.col), _p(val), _p(Bc), width,
                                              width, _p(out), width)
        return out
    rows = np.asarray(rows, dtype=np.int64)
    starts, ends = csr.rowptr[rows], csr.rowptr[rows + 1]
    idx = np.concatenate([np.arange(s, e) for s, e in zip(starts, ends)]) if rows.size else np.zeros(0, np.int64)
    rp = np.zeros(rows.size + 1, dtype=np.int64)
    rp[1:] = np.cumsum(ends - starts)
    sub = CSR(rp, np.ascontiguousarray(csr.col[idx]), np.ascontiguousarray(val[idx]))
    return spmm(sub, B)


def spmm_tiles(tl, Bblocks, width) -> np.ndarray:
    """P-way staged SpMM for one row block (bit-identical to spmm())."""
    P = len(tl)
    dt = Bblocks[0].dtype
    nrows = tl[0][0].shape[0] - 1
    rps = [np.ascontiguousarray(t[0].astype(np.int64)) for t in tl]
    cols = [np.ascontiguousarray(t[1].astype(np.int64)) for t in tl]
    vals = [np.ascontiguousarray(t[2].astype(dt)) for t in tl]
    Bs = [np.ascontiguousarray(b) for b in Bblocks]
    arr = lambda xs: (ctypes.c_void_p * P)(*[x.ctypes.data for x in xs])
    out = np.empty((nrows, width), dtype=dt)
    getattr(_L(), f"orc_spmm_tiles_{_suf(dt)}")(nrows, P, arr(rps), arr(cols), arr(vals), arr(Bs), width, width,
                                                _p(out), width)
    return out


def gemm(A, B, transA=False, transB=False) -> np.ndarray:
    """C = op(A)·op(B), fp64 acc in ascending k (Eq. 5, 10, 11)."""
    dt = A.dtype
    A = np.ascontiguousarray(A)
    B = np.ascontiguousarray(B.astype(dt))
    M = A.shape[1] if transA else A.shape[0]
    K = A.shape[0] if transA else A.shape[1]
    N = B.shape[0] if transB else B.shape[1]
    C = np.empty((M, N), dtype=dt)
    getattr(_L(), f"orc_gemm_{_suf(dt)}")(M, N, K, _p(A), A.shape[1], int(transA), _p(B), B.shape[1], int(transB),
                                          _p(C), N)
    return C


def softmax_ce(Z, y, ntrain):
    """Returns (loss_sum over labelled rows (fp64), G = dLoss/dZ with loss = sum / ntrain)."""
    Z = np.ascontiguousarray(Z)
    y = np.ascontiguousarray(y, dtype=np.int32)
    G = np.empty_like(Z)
    s = ctypes.c_double(0.0)
    getattr(_L(), f"orc_softmax_ce_{_suf(Z.dtype)}")(Z.shape[0], Z.shape[1], _p(Z), Z.shape[1], _p(y), ntrain,
                                                     _p(G), G.shape[1], ctypes.byref(s))
    return s.value, G


def adam(W, g, m, v, t, lr=0.01, b1=0.9, b2=0.999, eps=1e-8):
    """In-place Adam step t (>= 1) on contiguous arrays."""
    for a in (W, g, m, v):
        assert a.flags.c_contiguous
    getattr(_L(), f"orc_adam_{_suf(W.dtype)}")(W.size, _p(W), _p(g.astype(W.dtype)), _p(m), _p(v), t, lr, b1, b2, eps)


def relu(Z):
    """Eq. 7 with sigma = ReLU."""
    return np.maximum(Z, np.zeros((), Z.dtype))


def spmm_first(d_in, d_out) -> bool:
    """§4.4 order rule, reading C10: SpMM first iff d(l) < d(l+1)."""
    return d_in < d_out


# ------------------------------------------------------------------ epoch
@dataclass
class EpochResult:
    perm: np.ndarray
    Z: list                 # pre-activation outputs per layer (permuted order)
    logits: np.ndarray      # Z[L-1] (or ReLU(Z[L-1]) with relu_last)
    loss: float
    WG: list                # per-layer weight gradients
    W: list                 # weights after Adam
    m: list
    v: list
    T: list                 # Â'^T H_l for S-order layers (None otherwise)


def epoch(pg: PermutedGraph, X, y, Ws, relu_last=False, dtype=np.float32, lr=0.01, b1=0.9, b2=0.999, eps=1e-8,
          adam_state=None, t=1, P=1) -> EpochResult:
    """One full-batch epoch (Fig. 1): L forward layers (Eq. 5-7 with
    the §4.4 order rule), softmax-CE, L backward layers (Eq.
    8-11), weight-gradient sum and Adam.

    X (n x d0) and y (n) are in ORIGINAL vertex order and are permuted here
    (X'[perm[v]] = X[v]).  With P > 1 the SpMMs run in the P-way simulation
    mode (bit-identical) and W_G is the rank-ordered sum of per-rank partials.
    """
    n = pg.n
    L = len(Ws)
    X = np.asarray(X)
    Xp = np.empty((n, X.shape[1]), dtype=dtype)
    Xp[pg.perm] = X.astype(dtype)
    yp = np.empty(n, dtype=np.int32)
    yp[pg.perm] = y
    Ws = [np.ascontiguousarray(W.astype(dtype)) for W in Ws]
    p = partition_vector(n, P)

    tl_cache = {}

    def agg(direction, M):
        """Â'^T M (direction 'F', Eq. 6) or Â' M (direction 'B', Eq. 9)."""
        if P == 1:
            return spmm(pg.At if direction == "F" else pg.A, M)
        out = np.empty((n, M.shape[1]), dtype=dtype)
        blocks = [np.ascontiguousarray(M[p[j]:p[j + 1]]) for j in range(P)]
        for i in range(P):
            if (direction, i) not in tl_cache:
                tl_cache[(direction, i)] = tiles_dir(pg, P, i, direction)
            out[p[i]:p[i + 1]] = spmm_tiles(tl_cache[(direction, i)], blocks, M.shape[1])
        return out

    # ---- forward (Eq. 5-7; Eq. 12)
    H = [Xp]
    Z, T = [], []
    for l in range(L):
        if spmm_first(Ws[l].shape[0], Ws[l].shape[1]):
            Tl = agg("F", H[l])                    # Â'^T H
            Zl = gemm(Tl, Ws[l])                   # (Â'^T H) W
        else:
            Tl = None
            HW = gemm(H[l], Ws[l])                 # Eq. 5
            Zl = agg("F", HW)                      # Eq. 6
        Z.append(Zl)
        T.append(Tl)
        if l < L - 1 or relu_last:
            H.append(relu(Zl))                     # Eq. 7
        else:
            H.append(Zl)
    logits = H[L]

    # ---- loss
    ntrain = int((yp >= 0).sum())
    loss_sum, G = softmax_ce(logits, yp, max(ntrain, 1))
    loss = loss_sum / max(ntrain, 1)

    # ---- backward (Eq. 8-11)
    WG = [None] * L
    for l in range(L - 1, -1, -1):
        relu_here = (l < L - 1) or relu_last
        ZG = G * (Z[l] > 0).astype(dtype) if relu_here else G     # Eq. 8 (C3, C27)
        if T[l] is None:
            HWG = agg("B", ZG)                                       # Eq. 9
            WG[l] = _wgrad(H[l], HWG, p, P)                          # Eq. 10 (C2)
            if l > 0:
                G = gemm(HWG, Ws[l], transB=True)                    # Eq. 11
        else:
            WG[l] = _wgrad(T[l], ZG, p, P)
            if l > 0:
                G = agg("B", gemm(ZG, Ws[l], transB=True))

    # ---- Adam
    if adam_state is None:
        adam_state = ([np.zeros_like(W) for W in Ws], [np.zeros_like(W) for W in Ws])
    m = [np.ascontiguousarray(a.astype(dtype)).copy() for a in adam_state[0]]
    v = [np.ascontiguousarray(a.astype(dtype)).copy() for a in adam_state[1]]
    Wn = [W.copy() for W in Ws]
    for l in range(L):
        adam(Wn[l], np.ascontiguousarray(WG[l]), m[l], v[l], t, lr, b1, b2, eps)
    return EpochResult(pg.perm, Z, logits, loss, WG, Wn, m, v, T)


def _wgrad(H, G, p, P):
    """W_G = H^T G (Eq. 10, reading C2); P-way: rank-ordered sum of partials."""
    if P == 1:
        return gemm(H, G, transA=True)
    acc = None
    for i in range(P):
        part = gemm(np.ascontiguousarray(H[p[i]:p[i + 1]]), np.ascontiguousarray(G[p[i]:p[i + 1]]), transA=True)
        acc = part if acc is None else (acc + part).astype(part.dtype)
    return acc


def tiles_dir(pg, P, rank, direction):
    t = tiles(pg, P, rank)
    return t[direction]


# ------------------------------------------------- ReLU branch choices (reading C31)
def forward_preactivations(pg: PermutedGraph, Xp, Ws, relu_last=False):
    """The forward of oracle.epoch (Eq. 5-7, §4.4 order rule) on inputs already in permuted
    order, returning every layer's pre-activation Z_l and input H_l (fp32 storage).  The
    SpMMs are oracle.spmm (fp64 accumulation, ascending); the dense products use numpy's
    float64 matmul as the library primitive (SURVEY §8(c) allows a matmul as a step) and are
    rounded once to fp32, so a value can differ from oracle.gemm's only by fp64 rounding before
    that rounding.  Used at full size, where oracle.gemm's single-threaded loops take hours."""
    L = len(Ws)
    H = [np.ascontiguousarray(Xp, dtype=np.float32)]
    Z = []
    for l in range(L):
        W = np.asarray(Ws[l], dtype=np.float64)
        if spmm_first(W.shape[0], W.shape[1]):
            T = spmm(pg.At, H[l])
            Zl = (T.astype(np.float64) @ W).astype(np.float32)
        else:
            HW = (H[l].astype(np.float64) @ W).astype(np.float32)
            Zl = spmm(pg.At, HW)
        Z.append(Zl)
        H.append(relu(Zl) if (l < L - 1 or relu_last) else Zl)
    return Z, H


def backward_given_masks(pg: PermutedGraph, H, G, Ws, masks):
    """Exact (fp64) backward of Eq. 8-11 with the ReLU' decisions given: masks[l] is the
    boolean mask of layer l's ReLU (None for a linear layer), H[l] the layer inputs
    (H[0] = X'), G = dLoss/dlogits.  Returns W_G,l for every l (fp64).  With masks[l] =
    Z_l > 0 it is the plain backward of oracle.epoch (pinned against it and against torch
    autograd in tests/test_oracle_numerics.py); with another ReLU branch choice at
    pre-activations inside the fp32 error of 0 it is the exact gradient of that choice."""
    L = len(Ws)
    A64 = CSR(pg.A.rowptr, pg.A.col, pg.A.val.astype(np.float64))
    At64 = CSR(pg.At.rowptr, pg.At.col, pg.At.val.astype(np.float64))
    WG = [None] * L
    G = np.asarray(G, dtype=np.float64)
    for l in range(L - 1, -1, -1):
        W = np.asarray(Ws[l], dtype=np.float64)
        ZG = G * masks[l] if masks[l] is not None else G                 # Eq. 8 (C3, C27)
        Hl = np.asarray(H[l], dtype=np.float64)
        if not spmm_first(W.shape[0], W.shape[1]):
            HWG = spmm(A64, ZG)                                          # Eq. 9
            WG[l] = Hl.T @ HWG                                           # Eq. 10 (C2)
            if l > 0:
                G = HWG @ W.T                                            # Eq. 11
        else:
            T = spmm(At64, Hl)
            WG[l] = T.T @ ZG
            if l > 0:
                G = spmm(A64, ZG @ W.T)
    return WG
