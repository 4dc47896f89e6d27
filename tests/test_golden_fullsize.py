"""Provenance and shape checks of the full-size oracle goldens
(tests/golden/fullsize_<cfg>.npz, written by scripts/make_fullsize_golden.py
from oracle/ only; used by tests/test_gpu_fullsize_golden.py).  CPU only."""
import json
import os

import numpy as np

import gen

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    z = np.load(os.path.join(GOLDEN, f"fullsize_{name}.npz"), allow_pickle=False)
    return {k: z[k] for k in z.files}, json.loads(str(z["meta"]))


def test_golden_files_are_oracle_written():
    """The goldens carry their provenance (script, oracle configuration, host) and match the
    workload table; runs on CPU too (no GPU needed)."""
    for name in ("reddit", "products", "proteins"):
        g, meta = load_golden(name)
        w = gen.WORKLOADS[name]
        assert meta["script"].startswith("scripts/make_fullsize_golden.py")
        assert meta["n"] == w.n and meta["m"] == w.m and tuple(meta["dims"]) == w.dims
        assert g["rows"].shape[0] >= 8192 and np.all(np.diff(g["rows"]) > 0)
        assert g["logits_rows"].shape == (g["rows"].shape[0], w.dims[-1])
        for l in range(len(w.dims) - 1):
            assert g[f"WG{l}"].shape == (w.dims[l], w.dims[l + 1])
            # first Adam step from zero state (reading C6): m = (1 - b1) g, v = (1 - b2) g^2
            gg = g[f"WG{l}"].astype(np.float64)
            assert np.allclose(g[f"m{l}"], 0.1 * gg, rtol=1e-6, atol=1e-30)
            assert np.allclose(g[f"v{l}"], 0.001 * gg * gg, rtol=1e-5, atol=1e-37)
        assert np.isfinite(float(g["loss"])) and 0 < float(g["loss"]) < 2 * np.log(w.dims[-1])
