"""Calibrate bench.py's row-sampled oracle estimate against a FULL single-core oracle epoch.

The full-size goldens (scripts/make_fullsize_golden.py) time one complete oracle epoch per
config on one pinned core (meta "oracle_epoch_s").  On the same host, this script runs the
estimator bench.py uses for `cpu_baseline` / `--impl reference` (oracle_epoch_sample: every op
of one epoch on R sampled output rows, scaled by n/R), pinned the same way, and records
ratio = full / sampled in profiles/r02_oracle_calibration.json.  bench.py multiplies its
sampled estimate by that ratio and reports both numbers.

The estimate needs it: a few hundred sampled rows keep the strided K-sweeps of the oracle's
W_G = H^T HW_G products in cache, the full epoch does not.

usage: python scripts/calibrate_oracle.py reddit proteins products [--core 4]
"""
import argparse
import json
import os
import statistics
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import gen    # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="+")
    ap.add_argument("--core", type=int, default=4)
    a = ap.parse_args()
    os.sched_setaffinity(0, {a.core})
    path = os.path.join(ROOT, "profiles", "r02_oracle_calibration.json")
    out = json.load(open(path)) if os.path.exists(path) else {}
    for name in a.configs:
        z = np.load(os.path.join(ROOT, "tests", "golden", f"fullsize_{name}.npz"))
        meta = json.loads(str(z["meta"]))
        w = gen.WORKLOADS[name]
        rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
        R = bench.auto_rows(w)
        ests = [bench.oracle_epoch_sample(w, rp, col, R, seed=s)[0] for s in range(3)]
        est = statistics.median(ests)
        full_ms = meta["oracle_epoch_s"] * 1e3
        out[name] = {"full_epoch_ms": full_ms, "sampled_estimate_ms": est, "ratio": full_ms / est, "rows_sampled": R,
                     "host_cpu": meta["host_cpu"], "golden": f"tests/golden/fullsize_{name}.npz",
                     "how": "full = one complete single-core oracle epoch (scripts/make_fullsize_golden.py); "
                            "sampled = median of 3 bench.oracle_epoch_sample runs on the same host and core setup"}
        print(json.dumps({name: out[name]}), flush=True)
        json.dump(out, open(path, "w"), indent=1)


if __name__ == "__main__":
    main()
