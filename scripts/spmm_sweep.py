"""Time the staged SpMM alone (mggcn_debug_spmm) on a BASELINE workload for
kernel-variant sweeps.  Usage: python scripts/spmm_sweep.py [workload] [widths...]"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402
from paper_conf_icpp_balinsc22_b200 import GCN  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "reddit"
widths = [int(x) for x in sys.argv[2:]] or [256, 44]
w = gen.WORKLOADS[wl]
rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
gm = GCN(w.n, rp, col, None, (max(widths), max(widths)), perm_seed=int(os.environ.get('PERM_SEED', w.perm_seed)),
         flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
for width in widths:
    B = torch.randn((w.n, width), device="cuda")
    out = torch.empty((w.n, width), device="cuda")
    for d in (0, 1):
        mg.mggcn_debug_spmm(gm.m, d, B, width, width, out, width)
        torch.cuda.synchronize()
        gm.profile(reset=True)
        t = time.perf_counter()
        reps = 5
        for _ in range(reps):
            mg.mggcn_debug_spmm(gm.m, d, B, width, width, out, width)
        torch.cuda.synchronize()
        wall = (time.perf_counter() - t) * 1e3 / reps
        sp_ms, sp_n = gm.profile(reset=True)["spmm"]
        ms = sp_ms / max(sp_n, 1)
        gb = w.m * width * 4 / 1e9
        print(f"{wl} width {width} dir {d}: {ms:.3f} ms/launch (wall {wall:.3f})  gather {gb / ms:.1f} TB/s  "
              f"WIN={os.environ.get('MGGCN_SPMM_WIN', '512')} CARVE={os.environ.get('MGGCN_SPMM_CARVEOUT')} "
              f"PERM={os.environ.get('PERM_SEED')}", flush=True)
