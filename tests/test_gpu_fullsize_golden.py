"""End-to-end parity of ONE WHOLE EPOCH at BASELINE.json's full sizes
(north_star: "within max relative error 1e-3 ... on logits, loss and weight
gradients after one epoch, on the same synthetic inputs"; SURVEY.md §8(c)
"GPU-vs-oracle acceptance").

The expected values are tests/golden/fullsize_<cfg>.npz, written by
scripts/make_fullsize_golden.py, which calls ONLY oracle/ and gen/: one plain
unpartitioned oracle epoch (fp32 storage, fp64 accumulate, single core) on the
seeded inputs.  Nothing here feeds a GPU result into the oracle: the GPU runs
the whole epoch on its own (forward over all layers with the P-stage SpMM,
softmax-CE, backward, W_G reduction, Adam), in bench.py's launch
configuration, and is compared element by element with the oracle's:
  logits    on the golden's >= 8192 sampled rows (permuted ids, incl. the
            largest hub and zero-in-degree vertices)   rel <= 1e-3
  loss                                                  rel <= 1e-3
  W_G,l     every element, every layer                  rel <= 1e-3
  Adam m, v after the step, every element               rel <= 1e-3
  W after the step where |g| > 1e-3 max|g|, within
            1e-5 + lr |s(g_gpu) - s(g_ref)|, s(g) = g / (|g| + eps): the first
            Adam step is exactly W - lr s(g), ill-conditioned where |g| ~ eps
            (reading C30)
rel(x, r) = max|x - r| / max|r|.

ReLU branch choices (reading C31): where a pre-activation lies within the fp32
forward error of 0, both ReLU' decisions are correct fp32 results, and the gradients
below that ReLU (W_G,l, Adam m, v for l < L-1) depend on the choice; at Products-shaped
size a few hundred such decisions out of 6.3e8 move W_G,0 by ~1.4e-3 of its max (its
entries are sums of 2.45 M terms that largely cancel).  When such an entry misses 1e-3
against the golden, the test checks what is unique and that the rest is valid:
  (i)  every mask decision of the GPU that differs from an independent reference forward
       (oracle.forward_preactivations) sits at |Z_ref| <= 1e-6 max|Z_ref|, and they are
       at most 1e-6 of the entries;
  (ii) the entry is within 1e-3 of the exact fp64 backward at the GPU's branch choices
       (oracle.backward_given_masks, on the reference activations).
Partitioning is an exact re-organisation
(§8(c)), so the same golden serves P = 1 and the loopback P = 8 split of
north_star's 8-GPU target.  The inputs' fingerprints are checked first, so a
generator drift fails loudly instead of comparing different problems."""
import hashlib
import json
import os

import numpy as np
import pytest
import torch

import gen

pytestmark = pytest.mark.gpu
REL_TOL = 1e-3
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def rel(x, r):
    r = np.asarray(r, np.float64)
    return float(np.abs(np.asarray(x, np.float64) - r).max() / max(np.abs(r).max(), 1e-30))


def sha(a):
    return hashlib.sha256(np.ascontiguousarray(a).tobytes()).hexdigest()


def load_golden(name):
    path = os.path.join(GOLDEN, f"fullsize_{name}.npz")
    z = np.load(path, allow_pickle=False)
    return {k: z[k] for k in z.files}, json.loads(str(z["meta"]))


def check_inputs(meta, rp, col, X, y, Ws):
    assert sha(rp) == meta["sha_rowptr"] and sha(col) == meta["sha_col"], "graph generator drifted"
    assert sha(X) == meta["sha_X"] and sha(y) == meta["sha_y"], "feature / label generator drifted"
    assert [sha(W) for W in Ws] == meta["sha_W"], "weight generator drifted"


def w_excess(g_ref, g_gpu, W_gpu, W_ref, lr=0.01, eps=1e-8):
    """Reading C30: after Adam's first step from zero state W1 = W0 - lr g / (|g| + eps) exactly,
    so where |g_ref| > 1e-3 max|g_ref| the two W may differ by lr |s(g_gpu) - s(g_ref)| (plus
    fp32 rounding, 1e-5); returns the largest excess over that bound (<= 0 passes)."""
    gr, gg = np.asarray(g_ref, np.float64), np.asarray(g_gpu, np.float64)
    mask = np.abs(gr) > 1e-3 * np.abs(gr).max()
    bound = 1e-5 + lr * np.abs(gg / (np.abs(gg) + eps) - gr / (np.abs(gr) + eps))
    diff = np.abs(np.asarray(W_gpu, np.float64) - np.asarray(W_ref, np.float64))
    return float((diff - bound)[mask].max())


_BRANCH_CACHE = {}


def branch_reference(name, gm_masks):
    """Reading C31: the reference forward (oracle), the audit of the GPU's differing ReLU
    decisions, and the exact fp64 backward at the GPU's branch choices (W_G, m, v).
    Cached per (config, masks): the eager and the captured epoch make the same decisions."""
    key = (name, tuple(hashlib.sha256(np.packbits(m).tobytes()).hexdigest() for m in gm_masks))
    if key not in _BRANCH_CACHE:
        _BRANCH_CACHE[key] = _branch_reference(name, gm_masks)
    return _BRANCH_CACHE[key]


def _branch_reference(name, gm_masks):
    import oracle
    w = gen.WORKLOADS[name]
    rp, col, X, y, Ws = gen.make_inputs(w)
    pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
    Xp = np.empty_like(X); Xp[pg.perm] = X
    yp = np.empty_like(y); yp[pg.perm] = y
    del X
    Z, H = oracle.forward_preactivations(pg, Xp, Ws)
    L = len(Ws)
    audit, masks, Hc = [], [], [Xp]
    for l in range(L - 1):
        mref = Z[l] > 0
        flip = gm_masks[l] != mref
        mx = float(np.abs(Z[l]).max())
        worst = float(np.abs(Z[l][flip]).max() / mx) if flip.any() else 0.0
        audit.append({"layer": l, "flips": int(flip.sum()), "entries": int(flip.size), "max_abs_preact_at_flip": worst})
        assert worst <= 1e-6 and flip.sum() <= 1e-6 * flip.size, audit[-1]        # C31 (i)
        masks.append(gm_masks[l])
        Hc.append(np.where(gm_masks[l], Z[l], 0).astype(np.float32))
    masks.append(None)
    ntrain = int((yp >= 0).sum())
    _, G = oracle.softmax_ce(Z[L - 1].astype(np.float64), yp, ntrain)
    WGb = oracle.backward_given_masks(pg, Hc, G, Ws, masks)
    print(json.dumps({"branch_audit": audit}))
    return {"WG": WGb, "m": [0.1 * w_ for w_ in WGb], "v": [0.001 * w_ * w_ for w_ in WGb]}


def compare_epoch(g, L, loss, WG, adam, Wn, logits_rows=None, branch=None):
    out = {"loss": abs(loss - float(g["loss"])) / abs(float(g["loss"]))}
    if logits_rows is not None:
        out["logits"] = rel(logits_rows, g["logits_rows"])
    for l in range(L):
        out[f"WG{l}"] = rel(WG[l], g[f"WG{l}"])
        mo, ve, t = adam[l]
        assert t == 1
        out[f"m{l}"] = rel(mo, g[f"m{l}"])
        out[f"v{l}"] = rel(ve, g[f"v{l}"])
        out[f"W{l}_excess"] = w_excess(g[f"WG{l}"], WG[l], Wn[l], g[f"W{l}"])
    print(json.dumps(out))
    failing = [k for k, v in out.items() if v > (0.0 if k.endswith("_excess") else REL_TOL)]
    below_relu = {f"{p}{l}" for p in ("WG", "m", "v") for l in range(L - 1)}
    if failing and branch is not None and set(failing) <= below_relu:
        ref = branch()                                        # reading C31: (i) inside, (ii) here
        got = {"WG": WG, "m": [a[0] for a in adam], "v": [a[1] for a in adam]}
        rechk = {k: rel(got[k[:-1]][int(k[-1])], ref[k[:-1]][int(k[-1])]) for k in failing}
        print(json.dumps({"branch_choice_recheck": rechk}))
        for k, v in rechk.items():
            assert v <= REL_TOL, (k, v, out, rechk)
        return out
    for k in failing:
        raise AssertionError((k, out[k], out))
    return out


@pytest.mark.parametrize("name,P", [("reddit", 1), ("reddit", 8), ("proteins", 1), ("products", 1)])
def test_fullsize_epoch_matches_oracle_golden(name, P):
    """Eager epoch (the path bench.py's profile loop times), P = 1 or loopback P-stage."""
    import paper_conf_icpp_balinsc22_b200 as mg
    from paper_conf_icpp_balinsc22_b200 import GCN
    assert torch.cuda.is_available()
    g, meta = load_golden(name)
    w = gen.WORKLOADS[name]
    L = len(w.dims) - 1
    rp, col, X, y, Ws = gen.make_inputs(w)
    check_inputs(meta, rp, col, X, y, Ws)
    gm = GCN(w.n, rp, col, None, w.dims, P=P, perm_seed=w.perm_seed,
             flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE, loopback=P > 1)
    try:
        assert sha(np.asarray(gm.perm, np.int64)) == meta["sha_perm"]
        gm.set_weights(Ws)
        Xp, yp = gm.permute_rows(X), gm.permute_rows(y)
        del X
        Xd, yd = gm.device_inputs(Xp), torch.from_numpy(yp).cuda()
        logits = torch.empty((w.n, w.dims[-1]), dtype=torch.float32, device="cuda")
        loss = gm.forward(Xd, yd, want_loss=True, logits=logits)
        rows = torch.from_numpy(g["rows"]).cuda()
        lrows = logits.index_select(0, rows).cpu().numpy()
        masks = [mg.mggcn_debug_layer(gm.m, l, (w.n, w.dims[l + 1])) > 0 for l in range(L - 1)]   # ReLU decisions
        gm.backward()
        WG = gm.grads()
        gm.step(lr=0.01)
        compare_epoch(g, L, loss, WG, [gm.adam_state(l) for l in range(L)], gm.get_weights(), lrows,
                      branch=lambda: branch_reference(name, masks))
    finally:
        gm.close()


@pytest.mark.parametrize("name", ["reddit", "products"])
def test_fullsize_captured_epoch_matches_oracle_golden(name):
    """The headline path of bench.py (N = 1): one replay of the captured epoch
    (mggcn_epoch_capture / mggcn_epoch_replay) from fresh weights."""
    import paper_conf_icpp_balinsc22_b200 as mg
    from paper_conf_icpp_balinsc22_b200 import GCN
    g, meta = load_golden(name)
    w = gen.WORKLOADS[name]
    L = len(w.dims) - 1
    rp, col, X, y, Ws = gen.make_inputs(w)
    check_inputs(meta, rp, col, X, y, Ws)
    gm = GCN(w.n, rp, col, None, w.dims, P=1, perm_seed=w.perm_seed, flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
    try:
        gm.set_weights(Ws)
        Xd, yd = gm.device_inputs(gm.permute_rows(X)), torch.from_numpy(gm.permute_rows(y)).cuda()
        del X
        gm.capture_epoch(Xd, yd, lr=0.01)
        gm.replay_epoch(1)
        gm.synchronize()
        # the captured epoch's ReLU decisions: AHWB_l after the step holds Z_G,l, so re-run the
        # forward eagerly from the replay's starting weights (bitwise the same kernels)
        WG, adam, Wn, loss = gm.grads(), [gm.adam_state(l) for l in range(L)], gm.get_weights(), gm.loss()
        gm.set_weights(Ws)
        gm.forward(Xd, yd, want_loss=False)
        masks = [mg.mggcn_debug_layer(gm.m, l, (w.n, w.dims[l + 1])) > 0 for l in range(L - 1)]
        compare_epoch(g, L, loss, WG, adam, Wn, branch=lambda: branch_reference(name, masks))
    finally:
        gm.close()

