"""Dense-block probe: one staged SpMM (mggcn_debug_spmm, P = 1) of a BASELINE workload at
full size, timed with CUDA events for several MGGCN_DENSE_THR / MGGCN_DENSE_PIECES settings,
with the dense statistics of each model.  JSON lines on stdout.

usage: python scripts/dense_probe.py [--workload reddit] [--width 256] [--thr 0,0.01,0.03]
       [--pieces 3] [--reps 10]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="reddit")
    ap.add_argument("--width", type=int, nargs="+", default=[256])
    ap.add_argument("--thr", default="0,0.01,0.02,0.03,0.05,0.1")
    ap.add_argument("--pieces", default="3")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--dir", type=int, default=0)
    a = ap.parse_args()
    import numpy as np
    import torch

    import gen
    import paper_conf_icpp_balinsc22_b200 as mg
    from paper_conf_icpp_balinsc22_b200 import GCN
    w = gen.WORKLOADS[a.workload]
    t0 = time.time()
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    gen_s = time.time() - t0
    wmax = max(a.width)
    B = torch.from_numpy(gen.features(w.n, wmax, 99)).cuda()
    out = torch.empty((w.n, wmax), dtype=torch.float32, device="cuda")
    ref = None
    for pieces in a.pieces.split(","):
        for thr in a.thr.split(","):
            os.environ["MGGCN_DENSE_THR"] = thr
            os.environ["MGGCN_DENSE_PIECES"] = pieces
            t0 = time.time()
            gm = GCN(w.n, rp, col, None, (wmax, wmax), P=1, perm_seed=w.perm_seed, flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
            setup = time.time() - t0
            st = mg.mggcn_dense_stats(gm.m)
            for width in a.width:
                for _ in range(3):
                    mg.mggcn_debug_spmm(gm.m, a.dir, B, wmax, width, out, wmax)
                gm.synchronize()
                gm.profile(reset=True)
                ms = []
                for _ in range(a.reps):
                    mg.mggcn_debug_spmm(gm.m, a.dir, B, wmax, width, out, wmax)
                    gm.synchronize()
                    ms.append(gm.profile(reset=True)["spmm"][0])   # library events on its compute stream
                res = out[:, :width].double().cpu().numpy()
                err = None
                if thr == "0" and width == wmax:
                    ref = res
                elif ref is not None and width == wmax:
                    err = float(np.abs(res - ref).max() / np.abs(ref).max())
                print(json.dumps({"workload": a.workload, "dir": a.dir, "width": width, "thr": float(thr),
                                  "pieces": int(pieces), "ms_median": float(np.median(ms)), "ms_min": float(min(ms)),
                                  "stats": st, "block_frac": st["block_entries"] / max(st["entries"], 1),
                                  "rel_vs_thr0": err, "setup_s": round(setup, 1), "gen_s": round(gen_s, 1)}),
                      flush=True)
            gm.close()


if __name__ == "__main__":
    main()
