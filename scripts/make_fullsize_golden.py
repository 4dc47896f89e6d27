"""Write the full-size end-to-end parity goldens (tests/golden/fullsize_<cfg>.npz).

Calls ONLY oracle/ and gen/ (the seeded input generator): one plain
unpartitioned oracle epoch (fp32 storage, fp64 accumulate, single thread,
pinned to one core) on BASELINE.json's full-size configs, and stores what
SURVEY.md §8(c) O11 compares:
  loss
  W_G,l for every layer      (Eq. 10, reading C2)
  Adam m, v, W after step 1  (reading C6)
  logits on >= 8192 rows     (Eq. 5-7; rows in PERMUTED order, incl. the
                              largest hub and zero-in-degree vertices)
plus fingerprints of the inputs (so the GPU test can prove it regenerated the
same graph / features), the oracle's wall time per step and the host CPU.

The oracle is the plain definition, identical for every P (partitioning is an
exact re-organisation, §8(c)), so one golden serves P = 1 and loopback P = 8.

usage: python scripts/make_fullsize_golden.py reddit [--core 0]
"""
import argparse
import hashlib
import json
import os
import platform
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen      # noqa: E402
import oracle   # noqa: E402

N_SAMPLE = 8192


def sha(a):
    return hashlib.sha256(np.ascontiguousarray(a).tobytes()).hexdigest()


def cpu_model():
    try:
        out = subprocess.check_output(["lscpu"], text=True)
        for line in out.splitlines():
            if line.startswith("Model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return platform.processor()


def sample_rows(n, perm, deg_in, seed=11):
    """Permuted-order row ids: the largest hub, up to 4 zero-in-degree
    vertices, and N_SAMPLE uniform rows (fixed seed)."""
    hub = int(perm[int(np.argmax(deg_in))])
    zeros = perm[np.flatnonzero(deg_in == 0)[:4]].tolist()
    rng = np.random.default_rng(seed)
    rnd = rng.choice(n, min(N_SAMPLE, n), replace=False).tolist()
    return np.unique(np.array([hub] + zeros + rnd, dtype=np.int64))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", choices=["cora", "reddit", "products", "proteins"])
    ap.add_argument("--core", type=int, default=0)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    os.sched_setaffinity(0, {a.core})
    w = gen.WORKLOADS[a.config]
    L = len(w.dims) - 1
    t0 = time.time()
    rp, col, X, y, Ws = gen.make_inputs(w)
    t_gen = time.time() - t0

    t0 = time.time()
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    t_prep = time.time() - t0
    deg_in = np.bincount(col, minlength=w.n)          # in-degree in ORIGINAL ids (symmetric graph)

    t0 = time.time()
    res = oracle.epoch(pg, X, y, Ws)
    t_epoch = time.time() - t0

    R = sample_rows(w.n, pg.perm, deg_in)
    out = a.out or os.path.join(ROOT, "tests", "golden", f"fullsize_{a.config}.npz")
    meta = {
        "config": a.config, "n": w.n, "m": w.m, "dims": list(w.dims),
        "seeds": {"G": w.seed_G, "X": w.seed_X, "y": w.seed_y, "W": w.seed_W, "perm": w.perm_seed},
        "sha_rowptr": sha(rp), "sha_col": sha(col), "sha_X": sha(X), "sha_y": sha(y),
        "sha_W": [sha(W) for W in Ws], "sha_perm": sha(pg.perm),
        "oracle": "oracle.epoch, fp32 storage / fp64 accumulate, P = 1, lr 0.01, betas (0.9, 0.999), eps 1e-8, t = 1",
        "oracle_epoch_s": round(t_epoch, 2), "oracle_prep_s": round(t_prep, 2), "gen_s": round(t_gen, 2),
        "cores": 1, "affinity": sorted(os.sched_getaffinity(0)), "host_cpu": cpu_model(), "nproc": os.cpu_count(),
        "rows": "permuted-order ids: largest hub, zero-in-degree vertices, 8192 uniform (seed 11)",
        "script": "scripts/make_fullsize_golden.py (calls only oracle/ and gen/)",
    }
    arrs = {"loss": np.float64(res.loss), "rows": R, "logits_rows": res.logits[R].astype(np.float32),
            "meta": np.array(json.dumps(meta))}
    for l in range(L):
        arrs[f"WG{l}"] = res.WG[l].astype(np.float32)
        arrs[f"W{l}"] = res.W[l].astype(np.float32)
        arrs[f"m{l}"] = res.m[l].astype(np.float32)
        arrs[f"v{l}"] = res.v[l].astype(np.float32)
    np.savez_compressed(out, **arrs)
    print(json.dumps({"out": out, "loss": res.loss, **{k: meta[k] for k in ("oracle_epoch_s", "oracle_prep_s", "host_cpu")}}))


if __name__ == "__main__":
    main()
