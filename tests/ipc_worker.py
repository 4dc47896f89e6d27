"""One rank of the 2-process MGGCN_F_IPC parity test (tests/test_gpu_ipc.py).

usage: python tests/ipc_worker.py RANK WORLD PORT OUT.npz MODE
Both ranks may share one GPU (the test box has one); the IPC backend maps the
peer's workspace with cudaIpcOpenMemHandle either way.  MODE = device | host |
prefetch selects how X / y reach the library each step.
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402
from paper_conf_icpp_balinsc22_b200 import GCN  # noqa: E402
from paper_conf_icpp_balinsc22_b200.dist import ipc_exchange  # noqa: E402


def main():
    rank, world, port, out, mode = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3], sys.argv[4], sys.argv[5]
    steps = int(sys.argv[6]) if len(sys.argv) > 6 else 2
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    torch.cuda.set_device(rank % torch.cuda.device_count())
    n, m, dims, seed = 3001, 60000, (100, 64, 64, 7), 75
    if mode.endswith("_sorder"):     # SpMM-first layer 0: X itself is pulled by the peers
        dims = (8, 32, 32, 7)
        mode = mode[:-len("_sorder")]
    rp, col = gen.rmat_csr(n, m, 71)
    X = gen.features(n, dims[0], 72)
    y = gen.labels(n, dims[-1], 73, 200)
    Ws = [gen.glorot(dims[l], dims[l + 1], 74 + l) for l in range(len(dims) - 1)]
    gm = GCN(n, rp, col, None, dims, P=world, rank=rank, perm_seed=seed, flags=mg.MGGCN_F_OVERLAP, comm="ipc",
             ipc_exchange=ipc_exchange(dist))
    gm.set_weights(Ws)
    Xl, yl = gm.permute_rows(X), gm.permute_rows(y)
    logits = torch.empty((gm.rows, dims[-1]), dtype=torch.float32, device="cuda")
    res = {}
    if mode == "device":
        Xin, yin = torch.from_numpy(Xl).cuda(), torch.from_numpy(yl).cuda()
    else:
        Xin, yin = Xl, yl
    if mode == "prefetch" and dims[0] < dims[1]:
        # MGGCN_F_IPC + SpMM-first layer 0: prefetch double-buffering is refused (include/mggcn.h)
        try:
            gm.prefetch(Xin, yin)
            res["prefetch_refused"] = np.int64(0)
        except mg.MggcnError as e:
            res["prefetch_refused"] = np.int64(e.code == mg.MGGCN_EUNSUPPORTED)
        gm.close()
        np.savez(out, **res)
        dist.barrier()
        dist.destroy_process_group()
        return
    if mode == "prefetch":
        gm.prefetch(Xin, yin)
    for s in range(steps):
        if mode == "prefetch":
            loss = gm.forward(None, None, want_loss=True, logits=logits if s == 0 else None)
            if s + 1 < steps:
                gm.prefetch(Xin, yin)
        else:
            loss = gm.forward(Xin, yin, want_loss=True, logits=logits if s == 0 else None)
        res[f"loss{s}"] = np.float64(loss)
        if s == 0:
            res["logits"] = logits.cpu().numpy()
        gm.backward()
        for l, g in enumerate(gm.grads()):
            res[f"WG{s}_{l}"] = g
        gm.step(lr=0.01)
    for l, W in enumerate(gm.get_weights()):
        res[f"W{l}"] = W
    res["row0"], res["rows"], res["perm"] = np.int64(gm.row0), np.int64(gm.rows), gm.perm
    gm.close()
    np.savez(out, **res)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
