"""B200-native MG-GCN hot path (Balın, Sancak, Çatalyürek, ICPP '22).

Thin ctypes binding of the C ABI in include/mggcn.h (libmggcn.so, built
in-tree for sm_100a by ``build_mggcn.py``).  Functions
keep the C names; this module only marshals arguments.  Every step of the
path runs in the library's kernels; there is no CPU fallback: if the shared
library is missing, importing the binding raises.

PyTorch provides device memory (one workspace tensor per model), CUDA streams
and the torch.distributed process group used to share the NCCL unique id.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MGGCN_LIB") or os.path.join(_HERE, "libmggcn.so")

MGGCN_OK, MGGCN_EINVAL, MGGCN_ENOMEM, MGGCN_ECUDA, MGGCN_ENCCL, MGGCN_ESTATE, MGGCN_EUNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
MGGCN_F_OVERLAP, MGGCN_F_RELU_LAST, MGGCN_F_TF32X1, MGGCN_F_NO_BCAST, MGGCN_F_PROFILE = 1, 2, 4, 16, 32
MGGCN_F_NO_COALESCE = 64
MGGCN_F_CACHE_L0 = 128
MGGCN_F_IPC = 256
MGGCN_F_REPL2 = 512        # 1.5D, replication factor c = 2
MGGCN_F_REPLICA1 = 1024    # with MGGCN_F_REPL2, nlocal = 1: this process is replica 1
MGGCN_F_TIMELINE = 2048    # per-stage comm / compute event timeline (mggcn_get_timeline)
MGGCN_IPC_BLOB_BYTES = 128
PROFILE_CLASSES = ("spmm", "gemm", "loss", "adam", "bcast", "allreduce", "other", "dense")

EXPORTS = (
    "mggcn_last_error", "mggcn_version", "mggcn_load_csr", "mggcn_graph_info", "mggcn_partition",
    "mggcn_part_info", "mggcn_part_export_tile", "mggcn_part_inv_deg", "mggcn_workspace_bytes",
    "mggcn_model_create", "mggcn_nccl_unique_id", "mggcn_set_weights", "mggcn_get_weights", "mggcn_forward",
    "mggcn_backward", "mggcn_step", "mggcn_get_loss", "mggcn_get_grad", "mggcn_get_adam", "mggcn_set_adam",
    "mggcn_get_profile", "mggcn_epoch_work", "mggcn_graph_free", "mggcn_part_free", "mggcn_model_free",
    "mggcn_debug_spmm", "mggcn_debug_gemm", "mggcn_kernel_launch_count", "mggcn_reset_cache",
    "mggcn_prefetch", "mggcn_ipc_export", "mggcn_ipc_connect", "mggcn_debug_layer", "mggcn_epoch_capture",
    "mggcn_epoch_replay", "mggcn_debug_comm_delay", "mggcn_get_timeline",
    "mggcn_epoch_work_detail", "mggcn_timeline_enable", "mggcn_debug_poison", "mggcn_stage_groups", "mggcn_dense_stats",
)


class MggcnError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"mggcn error {code}: {msg}")
        self.code = code


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python build_mggcn.py` "
                          "(the CUDA library is the only implementation; there is no fallback)")
    try:  # make sure the NCCL that torch bundles is the one resolved
        import torch  # noqa: F401
    except Exception:
        pass
    lib = ctypes.CDLL(LIB_PATH)
    P, i64, i32, u32, u64, f32, sz, up = (ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32,
                                          ctypes.c_uint64, ctypes.c_float, ctypes.c_size_t, ctypes.c_size_t)
    sig = {
        "mggcn_last_error": ([], ctypes.c_char_p),
        "mggcn_version": ([], ctypes.c_int),
        "mggcn_load_csr": ([i64, i64, P, P, P, P], ctypes.c_int),
        "mggcn_graph_info": ([P, P, P, P, P, P], ctypes.c_int),
        "mggcn_partition": ([P, i32, i32, u64, P], ctypes.c_int),
        "mggcn_part_info": ([P, P, P, P, P, P, P], ctypes.c_int),
        "mggcn_part_export_tile": ([P, i32, i32, P, P, P], ctypes.c_int),
        "mggcn_part_inv_deg": ([P, P], ctypes.c_int),
        "mggcn_workspace_bytes": ([P, i32, i32, P, u32, P], ctypes.c_int),
        "mggcn_model_create": ([P, i32, i32, P, u32, P, P, sz, up, up, P], ctypes.c_int),
        "mggcn_nccl_unique_id": ([P], ctypes.c_int),
        "mggcn_ipc_export": ([P, P], ctypes.c_int),
        "mggcn_ipc_connect": ([P, P], ctypes.c_int),
        "mggcn_set_weights": ([P, i32, P], ctypes.c_int),
        "mggcn_get_weights": ([P, i32, P], ctypes.c_int),
        "mggcn_forward": ([P, P, i64, P, P, P], ctypes.c_int),
        "mggcn_backward": ([P], ctypes.c_int),
        "mggcn_step": ([P, f32, f32, f32, f32], ctypes.c_int),
        "mggcn_get_loss": ([P, P], ctypes.c_int),
        "mggcn_get_grad": ([P, i32, P], ctypes.c_int),
        "mggcn_get_adam": ([P, i32, P, P, P], ctypes.c_int),
        "mggcn_set_adam": ([P, i32, P, P, i64], ctypes.c_int),
        "mggcn_get_profile": ([P, P, P, i32], ctypes.c_int),
        "mggcn_get_timeline": ([P, i64, P, P, P, i32], ctypes.c_int),
        "mggcn_timeline_enable": ([P, i32], ctypes.c_int),
        "mggcn_debug_poison": ([P, i32], ctypes.c_int),
        "mggcn_stage_groups": ([P, P, i32], ctypes.c_int),
        "mggcn_dense_stats": ([P, P, i32], ctypes.c_int),
        "mggcn_epoch_work": ([P, P, P, P, P], ctypes.c_int),
        "mggcn_epoch_work_detail": ([P, P, i32], ctypes.c_int),
        "mggcn_graph_free": ([P], None),
        "mggcn_part_free": ([P], None),
        "mggcn_model_free": ([P], None),
        "mggcn_debug_spmm": ([P, i32, P, i64, i32, P, i64], ctypes.c_int),
        "mggcn_debug_layer": ([P, i32, P, i64], ctypes.c_int),
        "mggcn_debug_comm_delay": ([P, ctypes.c_uint64, i32], ctypes.c_int),
        "mggcn_debug_gemm": ([i32, i64, i64, i64, P, i64, P, i64, P, i64, u32, up], ctypes.c_int),
        "mggcn_kernel_launch_count": ([], ctypes.c_int64),
        "mggcn_reset_cache": ([P], ctypes.c_int),
        "mggcn_prefetch": ([P, P, i64, P], ctypes.c_int),
        "mggcn_epoch_capture": ([P, P, i64, P, f32, f32, f32, f32], ctypes.c_int),
        "mggcn_epoch_replay": ([P, i32], ctypes.c_int),
    }
    for name, (args, res) in sig.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = res
    return lib


_lib = _load()


def lib():
    return _lib


def _check(rc):
    if rc != MGGCN_OK:
        raise MggcnError(rc, _lib.mggcn_last_error().decode(errors="replace"))


def _ptr(a):
    """Address of a numpy array / torch tensor (host or device) or None."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()


def _out_handle():
    return ctypes.c_void_p()


# ------------------------------------------------------------ C-named calls
def mggcn_version() -> int:
    return _lib.mggcn_version()


def mggcn_load_csr(n, rowptr, colidx, vals=None):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    vals = None if vals is None else np.ascontiguousarray(vals, dtype=np.float32)
    h = _out_handle()
    _check(_lib.mggcn_load_csr(n, colidx.shape[0], _ptr(rowptr), _ptr(colidx), _ptr(vals), ctypes.byref(h)))
    return h


def mggcn_graph_info(g):
    n, nnz = ctypes.c_int64(), ctypes.c_int64()
    sym, unit = ctypes.c_int32(), ctypes.c_int32()
    _check(_lib.mggcn_graph_info(g, ctypes.byref(n), ctypes.byref(nnz), ctypes.byref(sym), ctypes.byref(unit), None))
    deg = np.empty(n.value, dtype=np.float32)
    _check(_lib.mggcn_graph_info(g, None, None, None, None, _ptr(deg)))
    return {"n": n.value, "nnz": nnz.value, "symmetric": bool(sym.value), "unit_weights": bool(unit.value),
            "deg": deg}


def mggcn_partition(g, nparts, rank, perm_seed):
    h = _out_handle()
    _check(_lib.mggcn_partition(g, nparts, rank, perm_seed, ctypes.byref(h)))
    return h


def mggcn_part_info(part, with_perm=True):
    P, rank, n = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int64()
    _check(_lib.mggcn_part_info(part, ctypes.byref(P), ctypes.byref(rank), ctypes.byref(n), None, None, None))
    p = np.empty(P.value + 1, dtype=np.int64)
    perm = np.empty(n.value, dtype=np.int64) if with_perm else None
    tnnz = np.empty(2 * P.value, dtype=np.int64)
    _check(_lib.mggcn_part_info(part, None, None, None, _ptr(p), _ptr(perm), _ptr(tnnz)))
    return {"P": P.value, "rank": rank.value, "n": n.value, "p": p, "perm": perm,
            "tile_nnz_F": tnnz[:P.value], "tile_nnz_B": tnnz[P.value:]}


def mggcn_part_export_tile(part, direction, j):
    info = mggcn_part_info(part, with_perm=False)
    rows = int(info["p"][info["rank"] + 1] - info["p"][info["rank"]])
    nnz = int((info["tile_nnz_F"] if direction == 0 else info["tile_nnz_B"])[j])
    rp = np.empty(rows + 1, dtype=np.int32)
    col = np.empty(max(nnz, 1), dtype=np.int32)
    val = np.empty(max(nnz, 1), dtype=np.float32)
    _check(_lib.mggcn_part_export_tile(part, direction, j, _ptr(rp), _ptr(col), _ptr(val)))
    return rp, col[:nnz], val[:nnz]


def mggcn_part_inv_deg(part):
    info = mggcn_part_info(part, with_perm=False)
    rows = int(info["p"][info["rank"] + 1] - info["p"][info["rank"]])
    out = np.empty(rows, dtype=np.float32)
    _check(_lib.mggcn_part_inv_deg(part, _ptr(out)))
    return out


def _parts_array(parts):
    arr = (ctypes.c_void_p * len(parts))(*[p.value if isinstance(p, ctypes.c_void_p) else p for p in parts])
    return arr


def mggcn_workspace_bytes(parts, dims, flags=0):
    dims_a = np.ascontiguousarray(dims, dtype=np.int32)
    out = ctypes.c_size_t()
    _check(_lib.mggcn_workspace_bytes(_parts_array(parts), len(parts), len(dims) - 1, _ptr(dims_a), flags,
                                      ctypes.byref(out)))
    return out.value


def mggcn_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_lib.mggcn_nccl_unique_id(buf))
    return buf.raw


def mggcn_ipc_export(m) -> bytes:
    buf = ctypes.create_string_buffer(MGGCN_IPC_BLOB_BYTES)
    _check(_lib.mggcn_ipc_export(m, buf))
    return buf.raw


def mggcn_ipc_connect(m, blobs):
    """blobs: the P exports in rank order."""
    raw = b"".join(blobs)
    if len(raw) != MGGCN_IPC_BLOB_BYTES * len(blobs):
        raise ValueError("mggcn_ipc_connect: each blob must be MGGCN_IPC_BLOB_BYTES long")
    buf = ctypes.create_string_buffer(raw, len(raw))
    _check(_lib.mggcn_ipc_connect(m, buf))


def mggcn_model_create(parts, dims, flags, nccl_id, workspace_ptr, ws_bytes, compute_stream, comm_stream):
    dims_a = np.ascontiguousarray(dims, dtype=np.int32)
    idbuf = None if nccl_id is None else ctypes.create_string_buffer(bytes(nccl_id), 128)
    h = _out_handle()
    _check(_lib.mggcn_model_create(_parts_array(parts), len(parts), len(dims) - 1, _ptr(dims_a), flags, idbuf,
                                   workspace_ptr, ws_bytes, compute_stream, comm_stream, ctypes.byref(h)))
    return h


def mggcn_set_weights(m, layer, W):
    W = np.ascontiguousarray(W, dtype=np.float32)
    _check(_lib.mggcn_set_weights(m, layer, _ptr(W)))


def mggcn_get_weights(m, layer, shape):
    W = np.empty(shape, dtype=np.float32)
    _check(_lib.mggcn_get_weights(m, layer, _ptr(W)))
    return W


def mggcn_forward(m, X, ldx, y, want_loss=True, logits=None):
    loss = ctypes.c_float()
    _check(_lib.mggcn_forward(m, _ptr(X), ldx, _ptr(y), ctypes.byref(loss) if want_loss else None, _ptr(logits)))
    return loss.value if want_loss else None


def mggcn_backward(m):
    _check(_lib.mggcn_backward(m))


def mggcn_prefetch(m, X, ldx, y):
    _check(_lib.mggcn_prefetch(m, _ptr(X), ldx, _ptr(y)))


def mggcn_reset_cache(m):
    _check(_lib.mggcn_reset_cache(m))


def mggcn_step(m, lr=0.01, beta1=0.9, beta2=0.999, eps=1e-8):
    _check(_lib.mggcn_step(m, lr, beta1, beta2, eps))


def mggcn_epoch_capture(m, X, ldx, y, lr=0.01, beta1=0.9, beta2=0.999, eps=1e-8):
    _check(_lib.mggcn_epoch_capture(m, _ptr(X), ldx, _ptr(y), lr, beta1, beta2, eps))


def mggcn_epoch_replay(m, epochs=1):
    _check(_lib.mggcn_epoch_replay(m, epochs))


def mggcn_get_loss(m):
    loss = ctypes.c_float()
    _check(_lib.mggcn_get_loss(m, ctypes.byref(loss)))
    return loss.value


def mggcn_get_grad(m, layer, shape):
    G = np.empty(shape, dtype=np.float32)
    _check(_lib.mggcn_get_grad(m, layer, _ptr(G)))
    return G


def mggcn_get_adam(m, layer, shape):
    mo = np.empty(shape, dtype=np.float32)
    ve = np.empty(shape, dtype=np.float32)
    t = ctypes.c_int64()
    _check(_lib.mggcn_get_adam(m, layer, _ptr(mo), _ptr(ve), ctypes.byref(t)))
    return mo, ve, t.value


def mggcn_set_adam(m, layer, mom, vel, t):
    mom = np.ascontiguousarray(mom, dtype=np.float32)
    vel = np.ascontiguousarray(vel, dtype=np.float32)
    _check(_lib.mggcn_set_adam(m, layer, _ptr(mom), _ptr(vel), t))


def mggcn_get_profile(m, reset=False):
    ms = (ctypes.c_double * len(PROFILE_CLASSES))()
    n = (ctypes.c_int64 * len(PROFILE_CLASSES))()
    _check(_lib.mggcn_get_profile(m, ms, n, 1 if reset else 0))
    return {c: (ms[i], n[i]) for i, c in enumerate(PROFILE_CLASSES)}


def mggcn_timeline_enable(m, on=True):
    _check(_lib.mggcn_timeline_enable(m, 1 if on else 0))


def mggcn_get_timeline(m, reset=True):
    """Per-op records since the last reset (MGGCN_F_TIMELINE): a list of dicts
    {cls, spmm, stage, rank, stream, t0, t1} (device ms from the first record)."""
    cnt = ctypes.c_int64()
    _check(_lib.mggcn_get_timeline(m, 0, None, None, ctypes.byref(cnt), 0))
    n = cnt.value
    meta = np.zeros((max(n, 1), 5), dtype=np.int32)
    t = np.zeros((max(n, 1), 2), dtype=np.float64)
    _check(_lib.mggcn_get_timeline(m, n, _ptr(meta), _ptr(t), ctypes.byref(cnt), 1 if reset else 0))
    return [dict(cls=PROFILE_CLASSES[meta[i, 0]], spmm=int(meta[i, 1]), stage=int(meta[i, 2]), rank=int(meta[i, 3]),
                 stream=int(meta[i, 4]), t0=float(t[i, 0]), t1=float(t[i, 1])) for i in range(n)]


def mggcn_epoch_work(m):
    vals = [ctypes.c_double() for _ in range(4)]
    _check(_lib.mggcn_epoch_work(m, *[ctypes.byref(v) for v in vals]))
    return dict(zip(("spmm_bytes", "spmm_gather_bytes", "gemm_flops", "bcast_bytes"), [v.value for v in vals]))


WORK_DETAIL_KEYS = ("spmm_bytes", "spmm_struct_bytes", "spmm_gather_bytes", "spmm_gather_raw_bytes", "gemm_flops",
                    "gemm_bytes", "bcast_bytes", "ce_bytes", "spmm_stages")


def mggcn_epoch_work_detail(m):
    out = (ctypes.c_double * 16)()
    k = _lib.mggcn_epoch_work_detail(m, out, 16)
    if k < 0:
        _check(k)
    return {name: out[i] for i, name in enumerate(WORK_DETAIL_KEYS[:k])}


def mggcn_stage_groups(m):
    """Remote blocks per SpMM launch ([] = one launch per stage)."""
    sizes = (ctypes.c_int32 * 16)()
    k = _lib.mggcn_stage_groups(m, sizes, 16)
    if k < 0:
        _check(k)
    return [int(sizes[i]) for i in range(k)]


DENSE_STATS_KEYS = ("blocks", "block_entries", "row_groups", "chunks", "entries")


def mggcn_dense_stats(m):
    """Dense blocks of the launched stage tiles (tensor-core part of the SpMM)."""
    out = (ctypes.c_int64 * 8)()
    k = _lib.mggcn_dense_stats(m, out, 8)
    if k < 0:
        _check(k)
    return {name: int(out[i]) for i, name in enumerate(DENSE_STATS_KEYS[:k])}


def mggcn_kernel_launch_count() -> int:
    return _lib.mggcn_kernel_launch_count()


def mggcn_graph_free(g):
    _lib.mggcn_graph_free(g)


def mggcn_part_free(p):
    _lib.mggcn_part_free(p)


def mggcn_model_free(m):
    _lib.mggcn_model_free(m)


def mggcn_debug_spmm(m, direction, B, ldb, width, out, ldo):
    _check(_lib.mggcn_debug_spmm(m, direction, _ptr(B), ldb, width, _ptr(out), ldo))


def mggcn_debug_comm_delay(m, seed, max_us):
    _check(_lib.mggcn_debug_comm_delay(m, seed, max_us))


def mggcn_debug_poison(m, on=1):
    """1: NaN-fill BC slots before they are filled; 2: also drop the broadcast waits (negative control)."""
    _check(_lib.mggcn_debug_poison(m, int(on)))


def mggcn_debug_layer(m, layer, shape):
    """Host copy (rows x d_{l+1}) of AHWB_l (see include/mggcn.h)."""
    out = np.empty(shape, dtype=np.float32)
    _check(_lib.mggcn_debug_layer(m, layer, _ptr(out), shape[1]))
    return out


def mggcn_debug_gemm(op, M, N, K, A, lda, B, ldb, C, ldc, flags=0, stream=0):
    _check(_lib.mggcn_debug_gemm(op, M, N, K, _ptr(A), lda, _ptr(B), ldb, _ptr(C), ldc, flags, stream))


from .model import GCN  # noqa: E402  (convenience wrapper; marshalling only)
