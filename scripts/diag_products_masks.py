"""Products-shaped: how many ReLU mask decisions differ between the GPU forward and a
reference forward (fp64 accumulation, rounded to fp32 like the oracle), and where."""
import json, os, sys, time
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen, oracle
import paper_conf_icpp_balinsc22_b200 as mg
from paper_conf_icpp_balinsc22_b200 import GCN

w = gen.WORKLOADS["products"]
d = w.dims
rp, col, X, y, Ws = gen.make_inputs(w)
gm = GCN(w.n, rp, col, None, d, perm_seed=w.perm_seed, flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
gm.set_weights(Ws)
Xp, yp = gm.permute_rows(X), gm.permute_rows(y)
gm.forward(gm.device_inputs(Xp), torch.from_numpy(yp).cuda(), want_loss=True)
H1 = mg.mggcn_debug_layer(gm.m, 0, (w.n, d[1]))
H2 = mg.mggcn_debug_layer(gm.m, 1, (w.n, d[2]))
gm.close()
pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
T0 = oracle.spmm(pg.At, Xp)                                   # fp32 storage, fp64 accumulation
Z0 = (T0.astype(np.float64) @ Ws[0].astype(np.float64)).astype(np.float32)
H1r = np.maximum(Z0, 0)
HW1 = (H1r.astype(np.float64) @ Ws[1].astype(np.float64)).astype(np.float32)
Z1 = oracle.spmm(pg.At, HW1)
H2r = np.maximum(Z1, 0)
out = {}
for name, Hg, Zr in (("H1", H1, Z0), ("H2", H2, Z1)):
    flip = (Hg > 0) != (Zr > 0)
    mx = float(np.abs(Zr).max())
    out[name] = {"elements": int(Zr.size), "mask_flips": int(flip.sum()),
                 "max_abs_preact_at_flip_over_max": float(np.abs(Zr[flip]).max() / mx) if flip.any() else 0.0,
                 "rel_err_active": float(np.abs(np.where(Zr > 0, Hg - Zr, 0)).max() / mx),
                 "abs_err_active_p99_over_max": float(np.quantile(np.abs(Hg - np.maximum(Zr, 0))[Zr > 0], 0.99) / mx)}
print(json.dumps(out), flush=True)
