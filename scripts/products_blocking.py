"""Products-shaped SpMM: does 2-D blocking (row blocks x column panels) or a narrower
column window lower the time of the width-256 gather from a 2.5 GB operand?

VERDICT r01 asked for column-panel x feature-window blocking of blocks larger than L2.
The library already has both knobs: the P-stage schedule IS row-block x column-panel
blocking (rank i's stage j = rows of block i x columns of block j), and MGGCN_SPMM_WIN
sets the column window.  So on one GPU, loopback P = 2, 4, 8 with MGGCN_F_NO_BCAST
(timing only: the exchange copies are skipped, every tile still runs) and the
one-launch-per-stage schedule (MGGCN_STAGE_GROUP=1) is the P x P blocked SpMM, each
launch gathering from an n/P-row panel (2.4 GB / P).  Results: SpMM ms per width-256
forward SpMM (sum over its launches; CUDA events), for each blocking and window.

usage: python scripts/products_blocking.py [--parts 1,2,4,8] [--wins 0,128,64]
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402
from paper_conf_icpp_balinsc22_b200 import GCN  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="products")
    ap.add_argument("--parts", default="1,2,4,8")
    ap.add_argument("--wins", default="0,128,64")
    ap.add_argument("--width", type=int, default=256)
    a = ap.parse_args()
    w = gen.WORKLOADS[a.workload]
    if "_PB_CHILD" not in os.environ:      # the window is read once per process: one child per config
        import subprocess
        for P in [int(x) for x in a.parts.split(",")]:
            for win in [int(x) for x in a.wins.split(",")]:
                env = dict(os.environ, _PB_CHILD=f"{P}:{win}")
                r = subprocess.run([sys.executable, __file__, "--workload", a.workload, "--parts", str(P), "--wins",
                                    str(win), "--width", str(a.width)], env=env, capture_output=True, text=True)
                sys.stdout.write(r.stdout)
                if r.returncode:
                    sys.stdout.write(json.dumps({"P": P, "win": win, "error": r.stderr[-800:]}) + "\n")
                sys.stdout.flush()
        return
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    g = mg.mggcn_load_csr(w.n, rp, col)
    os.environ["MGGCN_STAGE_GROUP"] = "1"
    width = a.width
    B = torch.randn((w.n, width), device="cuda")
    out = torch.empty((w.n, width), device="cuda")
    for P in [int(x) for x in a.parts.split(",")]:
        for win in [int(x) for x in a.wins.split(",")]:
            if win:
                os.environ["MGGCN_SPMM_WIN"] = str(win)
            else:
                os.environ.pop("MGGCN_SPMM_WIN", None)
            flags = mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE | (mg.MGGCN_F_NO_BCAST if P > 1 else 0)
            gm = GCN(w.n, None, None, None, (width, width), P=P, perm_seed=w.perm_seed, flags=flags,
                     loopback=P > 1, graph=g)
            mg.mggcn_debug_spmm(gm.m, 0, B, width, width, out, width)
            torch.cuda.synchronize()
            gm.profile(reset=True)
            reps = 5
            for _ in range(reps):
                mg.mggcn_debug_spmm(gm.m, 0, B, width, width, out, width)
            torch.cuda.synchronize()
            prof = gm.profile(reset=True)
            sp_ms, sp_n = prof["spmm"]
            print(json.dumps({"workload": a.workload, "P": P, "blocks": f"{P}x{P}", "win": win or "auto",
                              "width": width, "spmm_ms": sp_ms / reps, "launches": sp_n / reps,
                              "panel_MB": w.n / P * width * 4 / 2**20}), flush=True)
            gm.close()
    mg.mggcn_graph_free(g)


if __name__ == "__main__":
    main()
