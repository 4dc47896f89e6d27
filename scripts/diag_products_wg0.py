"""Diagnose the Products-shaped W_G parity gap vs the golden (W_G0 1.4e-3, W_G1 1.2e-3):
recompute the whole BACKWARD in fp64 (oracle SpMMs, numpy fp64 GEMMs) from the GPU's own
forward activations (so the ReLU masks are the GPU's), and compare with the GPU's and the
golden's W_G.  If fp64-backward-on-GPU-forward matches the GPU, the gap comes from the
forward (mask decisions near 0); if it matches the golden, from the GPU's backward arithmetic."""
import json, os, sys, time
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen, oracle
import paper_conf_icpp_balinsc22_b200 as mg
from paper_conf_icpp_balinsc22_b200 import GCN

w = gen.WORKLOADS["products"]
d = w.dims
rp, col, X, y, Ws = gen.make_inputs(w)
z = np.load(os.path.join(os.path.dirname(__file__), "..", "tests", "golden", "fullsize_products.npz"))
gm = GCN(w.n, rp, col, None, d, perm_seed=w.perm_seed, flags=mg.MGGCN_F_OVERLAP | mg.MGGCN_F_PROFILE)
gm.set_weights(Ws)
Xp, yp = gm.permute_rows(X), gm.permute_rows(y)
logits = torch.empty((w.n, d[-1]), dtype=torch.float32, device="cuda")
gm.forward(gm.device_inputs(Xp), torch.from_numpy(yp).cuda(), want_loss=True, logits=logits)
H1 = mg.mggcn_debug_layer(gm.m, 0, (w.n, d[1]))
H2 = mg.mggcn_debug_layer(gm.m, 1, (w.n, d[2]))
Zl = logits.cpu().numpy()
gm.backward()
WG = gm.grads()
gm.close()
rel = lambda a, r: float(np.abs(np.asarray(a, np.float64) - r).max() / np.abs(r).max())
t = time.time()
pg = oracle.permute_graph(w.n, rp, col, None, seed=w.perm_seed)
A64 = oracle.CSR(pg.A.rowptr, pg.A.col, pg.A.val.astype(np.float64))
At64 = oracle.CSR(pg.At.rowptr, pg.At.col, pg.At.val.astype(np.float64))
T0 = oracle.spmm(At64, Xp.astype(np.float64))
ntrain = int((yp >= 0).sum())
_, G = oracle.softmax_ce(Zl.astype(np.float64), yp, ntrain)                 # dLoss/dlogits from the GPU logits
W = [Wl.astype(np.float64) for Wl in Ws]
# layer 2 (G-order, linear): HW_G2 = A' G ; W_G2 = H2^T HW_G2 ; G1 = HW_G2 W2^T * [H2 > 0]
HWG2 = oracle.spmm(A64, G)
wg2 = H2.astype(np.float64).T @ HWG2
G1 = (HWG2 @ W[2].T) * (H2 > 0)
HWG1 = oracle.spmm(A64, G1)
wg1 = H1.astype(np.float64).T @ HWG1
Z0 = (HWG1 @ W[1].T) * (H1 > 0)                                            # layer 0 is S-order: W_G0 = T0^T Z_G0
wg0 = T0.T @ Z0
out = {"t_s": time.time() - t}
for l, wr in enumerate((wg0, wg1, wg2)):
    gold = z[f"WG{l}"].astype(np.float64)
    out[f"WG{l}"] = {"gpu_vs_golden": rel(WG[l], gold), "fp64bwd_on_gpu_fwd_vs_golden": rel(wr, gold),
                     "gpu_vs_fp64bwd_on_gpu_fwd": rel(WG[l], wr)}
print(json.dumps(out), flush=True)
