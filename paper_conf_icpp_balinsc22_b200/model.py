"""GCN: convenience wrapper over the C ABI (marshalling only).

Owns one graph -> partition(s) -> model chain, the torch workspace tensor and
the two CUDA streams (compute = stream 0, comm = stream 1 of P:929-933).
"""
from __future__ import annotations

import numpy as np

from . import (MGGCN_F_IPC, MGGCN_F_OVERLAP, MGGCN_F_REPL2, MGGCN_F_REPLICA1, mggcn_backward, mggcn_epoch_capture,
               mggcn_epoch_work_detail,
               mggcn_epoch_replay, mggcn_epoch_work, mggcn_forward, mggcn_get_adam, mggcn_get_grad, mggcn_get_loss, mggcn_get_profile, mggcn_get_weights, mggcn_graph_free,
               mggcn_ipc_connect, mggcn_ipc_export, mggcn_load_csr, mggcn_model_create, mggcn_model_free,
               mggcn_part_free, mggcn_part_info, mggcn_partition, mggcn_prefetch, mggcn_set_adam,
               mggcn_set_weights, mggcn_step, mggcn_workspace_bytes)


class GCN:
    """Full-batch GCN (Eq. 1-11) on one GPU rank, or all P ranks in loopback mode.

    rowptr/col/vals: CSR of A in ORIGINAL vertex ids.  dims = (d_0, ..., d_L).
    """

    def __init__(self, n, rowptr, col, vals, dims, P=1, rank=0, perm_seed=0, flags=MGGCN_F_OVERLAP,
                 loopback=False, nccl_id=None, device=None, graph=None, comm="nccl", ipc_exchange=None,
                 replicas=1):
        """comm = "nccl" (nccl_id from mggcn_nccl_unique_id, shared by the caller) or "ipc"
        (MGGCN_F_IPC: peers map each other's workspaces; ipc_exchange(blob) -> list of the P
        blobs in rank order, e.g. dist.ipc_exchange over torch.distributed).

        replicas = 2: 1.5D (MGGCN_F_REPL2).  P is then the TOTAL number of
        ranks (P/2 row blocks); `rank` = replica * P/2 + block.  In loopback the model's
        rows are the n permuted rows twice (replica 0 then replica 1)."""
        import torch
        self.torch = torch
        self.dims = tuple(int(d) for d in dims)
        self.L = len(self.dims) - 1
        self.P, self.rank, self.loopback = P, rank, loopback
        own_graph = graph is None
        if replicas not in (1, 2) or P % replicas:
            raise ValueError("replicas must be 1 or 2 and divide P")
        self.replicas = replicas
        Pb = P // replicas                                   # row blocks
        if replicas == 2:
            flags |= MGGCN_F_REPL2
            if not loopback and rank // Pb == 1:
                flags |= MGGCN_F_REPLICA1
        g = mggcn_load_csr(n, rowptr, col, vals) if own_graph else graph
        try:
            ranks = list(range(P)) if loopback else [rank]
            self.parts = [mggcn_partition(g, Pb, r % Pb, perm_seed) for r in ranks]
        finally:
            if own_graph:
                mggcn_graph_free(g)
        info = mggcn_part_info(self.parts[0])
        self.n, self.p, self.perm = info["n"], info["p"], info["perm"]
        self.row0 = 0 if loopback else int(self.p[rank % Pb])
        self.rows = n if loopback else int(self.p[rank % Pb + 1] - self.p[rank % Pb])
        self.device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.comm = "loopback" if loopback or P == 1 else comm
        if self.comm == "ipc":
            if ipc_exchange is None:
                raise ValueError("GCN(comm='ipc') needs ipc_exchange")
            flags |= MGGCN_F_IPC
            nccl_id = None
        self.ws_bytes = mggcn_workspace_bytes(self.parts, self.dims, flags)
        self.workspace = torch.empty(self.ws_bytes, dtype=torch.uint8, device=self.device)
        self.cs = torch.cuda.Stream(device=self.device)
        # the comm stream outranks compute: NCCL's kernels take SMs as the SpMM's blocks retire (SPMM_YIELD)
        self.ms = torch.cuda.Stream(device=self.device, priority=-1)
        self.m = mggcn_model_create(self.parts, self.dims, flags, nccl_id, self.workspace.data_ptr(), self.ws_bytes,
                                    self.cs.cuda_stream, self.ms.cuda_stream)
        if self.comm == "ipc":
            mggcn_ipc_connect(self.m, ipc_exchange(mggcn_ipc_export(self.m)))

    # ---------------------------------------------------------------- data
    @property
    def ld0(self):
        """Padded input row stride: a device X with this stride is read in place."""
        return (self.dims[0] + 7) // 8 * 8

    def device_inputs(self, X_local):
        """Device copy of X_local in the padded layout the library reads without copying."""
        torch = self.torch
        Xd = torch.zeros((X_local.shape[0], self.ld0), dtype=torch.float32, device=self.device)
        Xd[:, :X_local.shape[1]] = torch.as_tensor(X_local, device=self.device)
        return Xd

    def permute_rows(self, X):
        """Rows owned by this model of the permuted matrix X' (X'[perm[v]] = X[v])."""
        X = np.asarray(X)
        Xp = np.empty_like(X)
        Xp[self.perm] = X
        own = Xp[self.row0:self.row0 + self.rows]
        if self.loopback and self.replicas > 1:          # every replica holds the rows again
            own = np.concatenate([own] * self.replicas)
        return np.ascontiguousarray(own)

    def set_weights(self, Ws):
        for l, W in enumerate(Ws):
            mggcn_set_weights(self.m, l, W)

    def get_weights(self):
        return [mggcn_get_weights(self.m, l, (self.dims[l], self.dims[l + 1])) for l in range(self.L)]

    # ---------------------------------------------------------- hot path
    def prefetch(self, X_local, y_local):
        """Start the copy of the next forward's inputs (overlaps the current epoch)."""
        torch = self.torch
        if isinstance(X_local, torch.Tensor) and X_local.is_cuda:
            torch.cuda.current_stream(self.device).synchronize()
        self._pref = (X_local, y_local)          # keep the buffers alive until consumed
        mggcn_prefetch(self.m, X_local, X_local.shape[1], y_local)

    def forward(self, X_local, y_local, want_loss=True, logits=None):
        """X_local / y_local: numpy (host) or torch (device or pinned host) rows of X', y';
        X_local = None consumes the inputs of the last prefetch()."""
        torch = self.torch
        if X_local is None:
            loss = mggcn_forward(self.m, None, 0, None, want_loss, logits)
            self._pref = None
            if logits is not None:
                torch.cuda.current_stream(self.device).wait_stream(self.cs)
            return loss
        if isinstance(X_local, torch.Tensor) and X_local.is_cuda:
            self.cs.wait_stream(torch.cuda.current_stream(self.device))
        ldx = X_local.shape[1] if X_local.ndim == 2 else self.dims[0]
        if isinstance(X_local, np.ndarray):
            X_local = np.ascontiguousarray(X_local, dtype=np.float32)
            y_local = np.ascontiguousarray(y_local, dtype=np.int32)
        loss = mggcn_forward(self.m, X_local, ldx, y_local, want_loss, logits)
        if logits is not None:
            torch.cuda.current_stream(self.device).wait_stream(self.cs)
        return loss

    def backward(self):
        mggcn_backward(self.m)

    def step(self, lr=0.01, beta1=0.9, beta2=0.999, eps=1e-8):
        mggcn_step(self.m, lr, beta1, beta2, eps)

    def capture_epoch(self, X_local, y_local, lr=0.01, beta1=0.9, beta2=0.999, eps=1e-8):
        """Record one forward -> backward -> step epoch as a CUDA graph (device X/y, whose
        addresses the graph keeps: refill them in place between replays)."""
        torch = self.torch
        self.cs.wait_stream(torch.cuda.current_stream(self.device))
        self._graph_inputs = (X_local, y_local)   # keep the baked-in buffers alive
        ldx = X_local.shape[1] if X_local.ndim == 2 else self.dims[0]
        mggcn_epoch_capture(self.m, X_local, ldx, y_local, lr, beta1, beta2, eps)

    def replay_epoch(self, epochs=1):
        """Launch the captured epoch `epochs` times (asynchronous, on the compute stream)."""
        mggcn_epoch_replay(self.m, epochs)

    def loss(self):
        return mggcn_get_loss(self.m)

    def grads(self):
        return [mggcn_get_grad(self.m, l, (self.dims[l], self.dims[l + 1])) for l in range(self.L)]

    def adam_state(self, layer):
        return mggcn_get_adam(self.m, layer, (self.dims[layer], self.dims[layer + 1]))

    def set_adam_state(self, layer, mom, vel, t):
        mggcn_set_adam(self.m, layer, mom, vel, t)

    def profile(self, reset=False):
        return mggcn_get_profile(self.m, reset)

    def epoch_work(self):
        return mggcn_epoch_work(self.m)

    def epoch_work_detail(self):
        return mggcn_epoch_work_detail(self.m)

    def synchronize(self):
        self.cs.synchronize()
        self.ms.synchronize()

    def close(self):
        if getattr(self, "m", None) is not None:
            mggcn_model_free(self.m)
            self.m = None
        for p in getattr(self, "parts", []):
            mggcn_part_free(p)
        self.parts = []

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
