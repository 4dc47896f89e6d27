"""NEXT-3 ablations on one B200, one JSON line per result.

  1. permutation on/off (§5.2, Fig. 6/7): per-rank nnz balance of the 1D
     partition for P = 2, 4, 8 (host, exact) and the P = 1 epoch time;
  2. overlap on/off (§4.3, Fig. 8) in loopback P = 4 (broadcasts are device
     copies on the comm stream; it exercises the event schedule, not NVLink);
  3. duplicate coalescing on/off;
  4. average-degree sweep (§6.4, Fig. 9): Arxiv-shaped R-MAT (n = 169,343,
     m = 1,166,243 x k, 128 features, 2 layers hidden 256, 40 classes).

Usage: python scripts/ablations.py [--quick]
"""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402
from paper_conf_icpp_balinsc22_b200 import GCN  # noqa: E402


def emit(**kw):
    print(json.dumps(kw), flush=True)


def epoch_ms(gm, X, y, steps=5, warmup=2):
    Xd = torch.from_numpy(gm.permute_rows(X)).cuda()
    yd = torch.from_numpy(gm.permute_rows(y)).cuda()
    for _ in range(warmup):
        gm.forward(Xd, yd, want_loss=False)
        gm.backward()
        gm.step()
    gm.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(gm.cs)
    for _ in range(steps):
        gm.forward(Xd, yd, want_loss=False)
        gm.backward()
        gm.step()
    b.record(gm.cs)
    b.synchronize()
    return a.elapsed_time(b) / steps


def main():
    quick = "--quick" in sys.argv
    w = gen.WORKLOADS["reddit"]
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    X = gen.features(w.n, w.dims[0], w.seed_X)
    y = gen.labels(w.n, w.dims[-1], w.seed_y)
    Ws = [gen.glorot(w.dims[l], w.dims[l + 1], w.seed_W + l) for l in range(3)]
    g = mg.mggcn_load_csr(w.n, rp, col)

    # 1a. partition balance with / without the random permutation
    for P in (2, 4, 8):
        for seed in (0, w.perm_seed):
            rank_nnz, tiles = [], []
            for r in range(P):
                part = mg.mggcn_partition(g, P, r, seed)
                info = mg.mggcn_part_info(part, with_perm=False)
                rank_nnz.append(int(info["tile_nnz_F"].sum()))
                tiles.extend(int(t) for t in info["tile_nnz_F"])
                mg.mggcn_part_free(part)
            emit(ablation="partition_balance", workload="reddit", P=P, permuted=bool(seed),
                 rank_nnz_max_over_mean=max(rank_nnz) / (sum(rank_nnz) / P),
                 tile_nnz_max_over_mean=max(tiles) / (sum(tiles) / len(tiles)))

    # 1b. epoch time P = 1, permuted vs natural R-MAT order
    for seed in (w.perm_seed, 0):
        gm = GCN(w.n, rp, col, None, w.dims, perm_seed=seed, flags=mg.MGGCN_F_OVERLAP, graph=g)
        gm.set_weights(Ws)
        emit(ablation="permutation", workload="reddit", P=1, permuted=bool(seed), epoch_ms=epoch_ms(gm, X, y))
        gm.close()

    # 2. overlap on / off, loopback P = 4, with the per-stage timeline of one epoch (Fig. 8 analogue;
    #    the "broadcasts" are device copies on the comm stream, so this shows the schedule, not NVLink)
    import bench
    for flags in (mg.MGGCN_F_OVERLAP, 0):
        gm = GCN(w.n, rp, col, None, w.dims, P=4, perm_seed=w.perm_seed, flags=flags, loopback=True, graph=g)
        gm.set_weights(Ws)
        ms = epoch_ms(gm, X, y, steps=3, warmup=1)
        mg.mggcn_timeline_enable(gm.m, True)
        mg.mggcn_get_timeline(gm.m, reset=True)
        epoch_ms(gm, X, y, steps=1, warmup=0)
        tl = mg.mggcn_get_timeline(gm.m, reset=True)
        mg.mggcn_timeline_enable(gm.m, False)
        summ = bench.timeline_summary(tl, w.dims, gm.p, 0)
        emit(ablation="overlap", workload="reddit", P=4, mode="loopback", overlap=bool(flags), epoch_ms=ms,
             timeline={k: summ[k] for k in ("epoch_span_ms", "compute_busy_ms", "comm_busy_ms", "exposed_comm_ms",
                                            "exposed_comm_frac")},
             first_spmm_stages=[dict(cls=r["cls"], stage=r["stage"], rank=r["rank"], stream=r["stream"],
                                     t0=round(r["t0"], 4), t1=round(r["t1"], 4))
                                for r in tl if r["spmm"] == 0])
        gm.close()

    # 3. duplicate coalescing on / off
    for flags in (mg.MGGCN_F_OVERLAP, mg.MGGCN_F_OVERLAP | mg.MGGCN_F_NO_COALESCE):
        gm = GCN(w.n, rp, col, None, w.dims, perm_seed=w.perm_seed, flags=flags, graph=g)
        gm.set_weights(Ws)
        emit(ablation="coalesce", workload="reddit", P=1, coalesce=not (flags & mg.MGGCN_F_NO_COALESCE),
             epoch_ms=epoch_ms(gm, X, y))
        gm.close()
    mg.mggcn_graph_free(g)
    del X

    # 4. average-degree sweep (Fig. 9 analogue; R-MAT in place of BTER)
    n, m0, dims = 169343, 1166243, (128, 256, 40)
    Xa = gen.features(n, dims[0], 4242)
    ya = gen.labels(n, dims[-1], 4343)
    Wa = [gen.glorot(dims[l], dims[l + 1], 4444 + l) for l in range(2)]
    for k in ((1, 4, 16) if quick else (1, 2, 4, 8, 16, 32, 64, 128)):
        m = m0 * k
        m -= m % 2
        t = time.perf_counter()
        rpa, cola = gen.rmat_csr(n, m, 4141 + k)
        gm = GCN(n, rpa, cola, None, dims, perm_seed=4545, flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
        gm.set_weights(Wa)
        ms = epoch_ms(gm, Xa, ya)
        prof = gm.profile(reset=True)
        work = gm.epoch_work()
        sp_ms = prof["spmm"][0] / 7
        emit(ablation="degree_sweep", n=n, m=m, avg_degree=m / n, dims=list(dims), epoch_ms=ms,
             spmm_ms=sp_ms, spmm_gather_TBps=work["spmm_gather_bytes"] / (sp_ms * 1e-3) / 1e12 if sp_ms else None,
             setup_s=time.perf_counter() - t)
        gm.close()


if __name__ == "__main__":
    main()
