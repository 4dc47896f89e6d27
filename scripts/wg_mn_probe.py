"""Probe the MN-major wgrad variant: integer-exact W_G = A^T B (op 2) for the
descriptor / TMA-swizzle setting in the environment; prints the max error."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402

rng = np.random.default_rng(0)
res = []
for (M, N, K) in [(128, 64, 64), (300, 256, 1000), (602, 41, 5000)]:
    lda, ldb = (M + 3) // 4 * 4, (N + 3) // 4 * 4
    A = np.zeros((K, lda), np.float32); A[:, :M] = rng.integers(-8, 9, (K, M))
    B = np.zeros((K, ldb), np.float32); B[:, :N] = rng.integers(-8, 9, (K, N))
    ref = A[:, :M].astype(np.float64).T @ B[:, :N].astype(np.float64)
    C = torch.full((M, N), np.nan, device="cuda")
    try:
        mg.mggcn_debug_gemm(2, M, N, K, torch.from_numpy(A).cuda(), lda, torch.from_numpy(B).cuda(), ldb, C, N)
        torch.cuda.synchronize()
        got = C.cpu().numpy()
        res.append(f"{M}x{N}x{K}: maxerr {np.nanmax(np.abs(got - ref)) if np.isfinite(got).any() else 'nan'} "
                   f"nan {int(np.isnan(got).sum())} zero-frac {float((got == 0).mean()):.3f}")
    except Exception as e:
        res.append(f"{M}x{N}x{K}: ERROR {e}")
        break
print(os.environ.get("MGGCN_WG_DESC"), os.environ.get("MGGCN_WG_TMASW"), " | ".join(res), flush=True)
