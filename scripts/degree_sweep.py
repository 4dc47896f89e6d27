"""NEXT-3 (c): the paper's average-degree sweep (§6.4, Fig. 9) on one B200.

The paper scales the Arxiv graph's edges by k = 1, 2, ..., 128 at a fixed vertex count
(BTER; n = 169,343, 1.166 M edges), with 512 random features and 40 classes, and trains
the 2-layer GCN with a 512-neuron hidden layer; it reports the median of 10
generated graphs per scale and the speed-up of 2 to 8 GPUs.  Here R-MAT replaces BTER
(SURVEY §8(f) NEXT-3), the median is over 3 seeds, and, since a gpurun call has one GPU,
each P is measured as the SOLO per-rank compute of rank 0 (include/mggcn.h
MGGCN_F_NO_BCAST: the rank's tiles and stages, every collective skipped) next to the
NVLink bound of the broadcasts it skips (library work model / 900 GB/s).  The P-GPU epoch
is at least max(compute, NVLink) with perfect overlap, so
    speed-up bound(P) = T_1 / max(T_solo(P), T_nvlink(P)).

usage: python scripts/degree_sweep.py [--scales 1,2,4,...] [--seeds 3] [--parts 2,4,8]
Prints one JSON line per (scale, seed, P) and one summary line per scale (medians).
"""
import argparse
import json
import os
import statistics
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402
from paper_conf_icpp_balinsc22_b200 import GCN  # noqa: E402

N, M0, DIMS = 169343, 1166243, (512, 512, 40)


def epoch_ms(gm, Xd, yd, steps, warmup):
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
    ap = argparse.ArgumentParser()
    ap.add_argument("--scales", default="1,2,4,8,16,32,64,128")
    ap.add_argument("--seeds", type=int, default=3)
    ap.add_argument("--parts", default="2,4,8")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    a = ap.parse_args()
    scales = [int(x) for x in a.scales.split(",")]
    parts = [int(x) for x in a.parts.split(",")]
    X = gen.features(N, DIMS[0], 4242)
    y = gen.labels(N, DIMS[-1], 4343)
    Ws = [gen.glorot(DIMS[l], DIMS[l + 1], 4444 + l) for l in range(2)]
    for k in scales:
        m = M0 * k
        m -= m % 2
        rows = []
        for s in range(a.seeds):
            t = time.perf_counter()
            rp, col = gen.rmat_csr(N, m, 4100 + 37 * k + s)
            g = mg.mggcn_load_csr(N, rp, col)
            res = {"scale": k, "seed": s, "n": N, "m": m, "avg_degree": m / N, "dims": list(DIMS)}
            gm = GCN(N, rp, col, None, DIMS, perm_seed=4545 + s, flags=mg.MGGCN_F_OVERLAP, graph=g)
            gm.set_weights(Ws)
            Xd, yd = gm.device_inputs(gm.permute_rows(X)), torch.from_numpy(gm.permute_rows(y)).cuda()
            res["P1_ms"] = epoch_ms(gm, Xd, yd, a.steps, a.warmup)
            gm.close()
            del Xd, yd
            for P in parts:
                gs = GCN(N, None, None, None, DIMS, P=P, rank=0, perm_seed=4545 + s,
                         flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_NO_BCAST, graph=g)
                gs.set_weights(Ws)
                Xl = gs.permute_rows(X)
                Xd, yd = gs.device_inputs(Xl), torch.from_numpy(gs.permute_rows(y)).cuda()
                res[f"solo_P{P}_ms"] = epoch_ms(gs, Xd, yd, a.steps, a.warmup)
                res[f"nvlink_P{P}_ms"] = gs.epoch_work()["bcast_bytes"] / 900e9 * 1e3
                res[f"speedup_bound_P{P}"] = res["P1_ms"] / max(res[f"solo_P{P}_ms"], res[f"nvlink_P{P}_ms"])
                gs.close()
                del Xd, yd
            mg.mggcn_graph_free(g)
            res["setup_and_run_s"] = time.perf_counter() - t
            print(json.dumps(res), flush=True)
            rows.append(res)
        summ = {"summary": True, "scale": k, "avg_degree": m / N, "seeds": a.seeds,
                "P1_ms_median": statistics.median(r["P1_ms"] for r in rows)}
        for P in parts:
            for key in (f"solo_P{P}_ms", f"nvlink_P{P}_ms", f"speedup_bound_P{P}"):
                summ[key + "_median"] = statistics.median(r[key] for r in rows)
        print(json.dumps(summ), flush=True)


if __name__ == "__main__":
    main()
