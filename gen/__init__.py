"""Seeded synthetic-input generators shared by the oracle and the CUDA path.

Holds none of the method's arithmetic: only Philox4x32-10 draws and the
assembly of the input CSR / features / labels / weights (recipe: SURVEY.md
§8(d) "Synthetic inputs", restated in DESIGN.md §3).  The C core lives in
gen/gen.c and is built to gen/libmggcn_gen.so.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libmggcn_gen.so")
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", src, "-o", _SO, "-lm"])
    return _SO


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        i64, u64, i32 = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int32
        lib.gen_philox4x32.argtypes = [ctypes.c_int, P, P, P]
        lib.gen_uniform.argtypes = [u64, u64, i64, P]
        lib.gen_features.argtypes = [i64, i64, i64, u64, P]
        lib.gen_labels.argtypes = [i64, i32, u64, i32, P]
        lib.gen_glorot.argtypes = [i64, i64, u64, P]
        lib.gen_rmat_pairs.argtypes = [i64, i64, u64, P, P]
        lib.gen_rmat_pairs.restype = i64
        lib.gen_rmat_csr.argtypes = [i64, i64, u64, P, P]
        lib.gen_rmat_csr.restype = i64
        _lib = lib
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def philox4x32(ctr, key, rounds: int = 10) -> np.ndarray:
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    _L().gen_philox4x32(rounds, _p(c), _p(k), _p(out))
    return out


def uniform(seed: int, start: int, count: int) -> np.ndarray:
    out = np.empty(count, dtype=np.float64)
    _L().gen_uniform(seed, start, count, _p(out))
    return out


def features(n: int, d: int, seed: int, ld: int | None = None) -> np.ndarray:
    ld = d if ld is None else ld
    X = np.empty((n, ld), dtype=np.float32)
    _L().gen_features(n, d, ld, seed, _p(X))
    return X


def labels(n: int, C: int, seed: int, unlabelled_per_mille: int = 0) -> np.ndarray:
    y = np.empty(n, dtype=np.int32)
    _L().gen_labels(n, C, seed, unlabelled_per_mille, _p(y))
    return y


def glorot(din: int, dout: int, seed: int) -> np.ndarray:
    W = np.empty((din, dout), dtype=np.float32)
    _L().gen_glorot(din, dout, seed, _p(W))
    return W


def rmat_pairs(n: int, npairs: int, seed: int):
    U = np.empty(max(npairs, 1), dtype=np.int32)
    V = np.empty(max(npairs, 1), dtype=np.int32)
    used = _L().gen_rmat_pairs(n, npairs, seed, _p(U), _p(V))
    if used < 0:
        raise MemoryError("gen_rmat_pairs failed")
    return U[:npairs], V[:npairs], used


def rmat_csr(n: int, m: int, seed: int):
    """Symmetric R-MAT CSR (rowptr int64[n+1], col int32[m]); duplicates kept."""
    rowptr = np.empty(n + 1, dtype=np.int64)
    col = np.empty(max(m, 1), dtype=np.int32)
    used = _L().gen_rmat_csr(n, m, seed, _p(rowptr), _p(col))
    if used < 0:
        raise ValueError(f"gen_rmat_csr failed (n={n}, m={m}: m must be even, n >= 2)")
    return rowptr, col[:m]


# --------------------------------------------------------------- workloads
@dataclass(frozen=True)
class Workload:
    """One BASELINE.json config (shapes per SURVEY.md §8.0)."""
    key: int          # config index k in 1..5 (seeds are 1000k + {1..5})
    name: str
    n: int
    m: int
    dims: tuple

    @property
    def seed_G(self): return 1000 * self.key + 1

    @property
    def seed_X(self): return 1000 * self.key + 2

    @property
    def seed_y(self): return 1000 * self.key + 3

    @property
    def seed_W(self): return 1000 * self.key + 4

    @property
    def perm_seed(self): return 1000 * self.key + 5


WORKLOADS = {
    "cora": Workload(1, "cora", 2708, 10556, (1433, 16, 7)),
    "reddit": Workload(2, "reddit", 232965, 114615892, (602, 256, 256, 41)),
    "products": Workload(3, "products", 2449029, 123718280, (100, 256, 256, 47)),
    "proteins": Workload(4, "proteins", 132534, 79122504, (8, 128, 128, 112)),
    "papers": Workload(5, "papers", 111059956, 3231371744, (128, 256, 256, 172)),
}


def make_inputs(w: Workload, unlabelled_per_mille: int = 0):
    """Graph (original vertex ids), X, y, [W_l] for a workload."""
    rowptr, col = rmat_csr(w.n, w.m, w.seed_G)
    X = features(w.n, w.dims[0], w.seed_X)
    y = labels(w.n, w.dims[-1], w.seed_y, unlabelled_per_mille)
    Ws = [glorot(w.dims[l], w.dims[l + 1], w.seed_W + l) for l in range(len(w.dims) - 1)]
    return rowptr, col, X, y, Ws


def glorot_bound(din: int, dout: int) -> float:
    return math.sqrt(6.0 / (din + dout))
