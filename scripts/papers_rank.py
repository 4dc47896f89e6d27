"""Papers-shaped (configs[4]) per-rank compute time on ONE GPU: rank R of the P = 8 1D partition.

BASELINE configs[4] is ogbn-papers100M-shaped (n = 111,059,956, m = 3,231,371,744, 128-256-256-172)
on 8 GPUs.  gpurun gives one GPU, and loopback would need all 8 ranks' ~100 GB on it, so this
runs ONE rank of the 8-way partition in the library's SOLO timing mode (MGGCN_F_NO_BCAST with
P > 1, nlocal = 1, no NCCL id; include/mggcn.h): the rank's own tiles, its share of every SpMM
stage (the remote stages gather from zeroed BC1/BC2 blocks of the right size), its GEMMs, CE
and Adam, with every collective skipped.  Results are invalid by construction; the number is
the rank's compute time per epoch.  The communication it skips is reported as a bound from
the library's own work model: broadcast bytes per rank / NVLink 900 GB/s.

The graph is the shared R-MAT generator at the full Papers shape (3.23 B non-zeros, ~13 GB of
int32 column indices on the host).  X and y of the rank's rows are seeded generator draws (not
tied to vertex ids: timing only).

usage: python scripts/papers_rank.py [--rank 0] [--parts 8] [--steps 5] [--warmup 2]
"""
import argparse
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def local_tile_check(gm, mg, w, rp, col, rank):
    """Correctness at full size on sampled rows (SOLO mode): mggcn_debug_spmm returns the rank's
    LOCAL tile times B (remote BC slots are never filled), i.e. for local row r (new id v):
    inv_deg(v) * sum over in-neighbours u of v with new id in this rank's block of B[u - p0]
    (Eq. 2 and Eq. 6 restricted to the diagonal tile).  The reference is computed in
    fp64 from the ORIGINAL CSR and the permutation (symmetric graph: in-neighbours = the row),
    independently of the library's partitioner and tiles."""
    import numpy as np
    import torch

    import gen
    p0, p1 = int(gm.p[rank]), int(gm.p[rank + 1])
    rows = p1 - p0
    width = 64
    B = torch.from_numpy(gen.features(rows, width, 777)).cuda()
    outd = torch.empty((rows, width), dtype=torch.float32, device="cuda")
    mg.mggcn_debug_spmm(gm.m, 0, B, width, width, outd, width)
    perm = np.asarray(gm.perm, dtype=np.int64)
    inv = np.empty_like(perm)
    inv[perm] = np.arange(perm.shape[0], dtype=np.int64)
    deg = np.diff(rp)
    local_orig = inv[p0:p1]
    ldeg = deg[local_orig]
    rng = np.random.default_rng(5)
    sample = set(rng.choice(rows, 254, replace=False).tolist())
    sample.add(int(np.argmax(ldeg)))
    z = np.flatnonzero(ldeg == 0)
    if z.size:
        sample.add(int(z[0]))
    sample = np.array(sorted(sample), dtype=np.int64)
    got = outd[torch.from_numpy(sample).cuda()].cpu().numpy().astype(np.float64)
    Bh = B.cpu().numpy()
    exp = np.zeros_like(got)
    for i, r in enumerate(sample):
        x = local_orig[r]
        nb = perm[col[rp[x]:rp[x + 1]].astype(np.int64)]
        nb = nb[(nb >= p0) & (nb < p1)] - p0
        d = np.float32(deg[x])
        s = Bh[nb].astype(np.float64).sum(axis=0)
        exp[i] = s * (np.float32(1.0) / d if d != 0 else 0.0)
    rel = float(np.abs(got - exp).max() / max(np.abs(exp).max(), 1e-30))
    return {"rows_checked": int(sample.size), "largest_local_in_degree": int(ldeg.max()),
            "rel_err": rel, "ok": rel <= 1e-4,
            "how": "mggcn_debug_spmm in SOLO mode = local tile x B; reference from the original CSR + perm (fp64)"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rank", type=int, default=0)
    ap.add_argument("--parts", type=int, default=8)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--workload", default="papers")
    ap.add_argument("--check", action="store_true",
                    help="after timing: the local-tile SpMM on sampled rows against the original CSR (host, fp64)")
    ap.add_argument("--timeline", action="store_true",
                    help="also record one epoch with MGGCN_F_TIMELINE and report per-SpMM stage sums / spans / gaps")
    args = ap.parse_args()

    import numpy as np
    import torch

    import gen
    import paper_conf_icpp_balinsc22_b200 as mg
    from paper_conf_icpp_balinsc22_b200 import GCN

    w = gen.WORKLOADS[args.workload]
    try:
        mem = subprocess.run(["free", "-g"], capture_output=True, text=True).stdout.split("\n")[1]
    except Exception:
        mem = "?"
    print("[papers_rank] host memory:", mem, flush=True)
    torch.cuda.set_device(0)
    t0 = time.perf_counter()
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    t_gen = time.perf_counter() - t0
    deg = np.diff(rp)
    print(f"[papers_rank] generated n={w.n} nnz={len(col)} in {t_gen:.1f} s; max deg {int(deg.max())}", flush=True)
    t0 = time.perf_counter()
    graph = mg.mggcn_load_csr(w.n, rp, col)
    t_load = time.perf_counter() - t0
    if not args.check:
        del rp, col
    print(f"[papers_rank] load_csr {t_load:.1f} s", flush=True)
    flags = mg.MGGCN_F_OVERLAP | mg.MGGCN_F_NO_BCAST | mg.MGGCN_F_PROFILE
    t0 = time.perf_counter()
    gm = GCN(w.n, None, None, None, w.dims, P=args.parts, rank=args.rank, perm_seed=w.perm_seed, flags=flags,
             graph=graph)
    t_part = time.perf_counter() - t0
    mg.mggcn_graph_free(graph)
    rows = gm.rows
    print(f"[papers_rank] partition + model {t_part:.1f} s; rank rows {rows}; workspace {gm.ws_bytes / 2**30:.1f} GiB",
          flush=True)
    Ws = [gen.glorot(w.dims[l], w.dims[l + 1], w.seed_W + l) for l in range(len(w.dims) - 1)]
    gm.set_weights(Ws)
    Xl = gen.features(rows, w.dims[0], w.seed_X)
    yl = gen.labels(rows, w.dims[-1], w.seed_y)
    Xd = gm.device_inputs(Xl)
    yd = torch.from_numpy(yl).cuda()
    del Xl
    torch.cuda.synchronize()

    def epoch():
        gm.forward(Xd, yd, want_loss=False)
        gm.backward()
        gm.step(lr=0.01)

    for _ in range(args.warmup):
        epoch()
    gm.synchronize()
    gm.profile(reset=True)
    tl_summary = None
    if args.timeline:
        mg.mggcn_timeline_enable(gm.m, True)      # one extra epoch, after the timed ones' warm-up
        mg.mggcn_get_timeline(gm.m, reset=True)
        epoch()
        gm.synchronize()
        tl = mg.mggcn_get_timeline(gm.m, reset=True)
        mg.mggcn_timeline_enable(gm.m, False)
        gm.profile(reset=True)
        comp = [r for r in tl if r["stream"] == 0]
        t_end = max(r["t1"] for r in comp)
        per = {}
        for r in comp:
            if r["cls"] != "spmm" or r["spmm"] < 0:
                continue
            d = per.setdefault(r["spmm"], {"stages": 0, "busy_ms": 0.0, "t0": r["t0"], "t1": r["t1"]})
            d["stages"] += 1
            d["busy_ms"] += r["t1"] - r["t0"]
            d["t0"] = min(d["t0"], r["t0"])
            d["t1"] = max(d["t1"], r["t1"])
        for d in per.values():
            d["span_ms"] = d["t1"] - d["t0"]
            d["gap_ms"] = d["span_ms"] - d["busy_ms"]
        busy = sum(r["t1"] - r["t0"] for r in comp)
        tl_summary = {"epoch_span_ms": t_end, "compute_busy_ms": busy, "compute_idle_ms": t_end - busy,
                      "spmm": {k: {kk: round(vv, 4) for kk, vv in v.items() if kk not in ("t0", "t1")}
                               for k, v in sorted(per.items())},
                      "stage_ms": [round(r["t1"] - r["t0"], 4) for r in comp if r["cls"] == "spmm"]}
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(gm.cs)
    for _ in range(args.steps):
        epoch()
    e1.record(gm.cs)
    e1.synchronize()
    gm.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    prof = gm.profile(reset=True)
    work = gm.epoch_work()
    bcast_ms = work["bcast_bytes"] / 900e9 * 1e3
    out = {
        "what": f"{w.name}-shaped rank {args.rank} of P = {args.parts}, SOLO timing mode (collectives skipped; "
                "results invalid): per-rank compute ms per epoch",
        "n": w.n, "nnz": w.m, "dims": list(w.dims), "rank_rows": int(rows),
        "compute_ms_per_epoch": ms,
        "stage_groups": mg.mggcn_stage_groups(gm.m),
        "dense": dict(mg.mggcn_dense_stats(gm.m), thr=os.environ.get("MGGCN_DENSE_THR", "default"),
                      min_rows=os.environ.get("MGGCN_DENSE_MIN_ROWS", "default")),
        "breakdown_ms_per_epoch": {k: v[0] / args.steps for k, v in prof.items()},
        "workspace_GiB": gm.ws_bytes / 2**30,
        "device_mem_reserved_GiB": torch.cuda.memory_reserved() / 2**30,
        "work_model": work,
        "bcast_bound_ms": bcast_ms,
        "bcast_note": "broadcast bytes received per rank per epoch (library work model) / 900 GB/s NVLink; "
                      "the 8-GPU epoch is at least max(compute, this) with perfect overlap",
        "setup_s": {"generate": t_gen, "load_csr": t_load, "partition+model": t_part},
        "steps": args.steps, "warmup": args.warmup, "timeline": tl_summary,
        "gpu": torch.cuda.get_device_name(0),
    }
    if args.check:
        out["check"] = local_tile_check(gm, mg, w, rp, col, args.rank)
    print(json.dumps(out), flush=True)
    gm.close()


if __name__ == "__main__":
    main()
