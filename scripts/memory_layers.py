"""NEXT-3 (d) (Fig. 12 of the paper): how many GCN layers (hidden
256) fit in one B200's 180 GB at P = 1, 2, 4, 8, from the library's own
buffer plan (mggcn_workspace_bytes of rank 0; host-only, no GPU needed).
The plan is the paper's L + 3 buffer scheme (§4.2): one AHWB per
layer plus shared HWB / BC1 / BC2, so bytes grow linearly in L.
Usage: python scripts/memory_layers.py > profiles/r01_memory_layers.jsonl"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_icpp_balinsc22_b200 as mg  # noqa: E402

HBM = 180e9          # B200 HBM3e per GPU (bytes)
RESERVE = 4e9        # CUDA context, NCCL buffers, allocator slack
for name in ("reddit", "products", "proteins"):
    w = gen.WORKLOADS[name]
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    g = mg.mggcn_load_csr(w.n, rp, col)
    del rp, col
    for P in (1, 2, 4, 8):
        part = mg.mggcn_partition(g, P, 0, w.perm_seed)
        size = {}
        for L in (2, 3, 4):
            dims = [w.dims[0]] + [256] * (L - 1) + [w.dims[-1]]
            flags = mg.MGGCN_F_OVERLAP
            size[L] = mg.mggcn_workspace_bytes([part], dims, flags)
        inc = size[4] - size[3]
        lmax = 3 + int((HBM - RESERVE - size[3]) // inc)
        print(json.dumps({"ablation": "memory_layers", "workload": name, "P": P, "hidden": 256,
                          "workspace_GB": {str(k): round(v / 1e9, 3) for k, v in size.items()},
                          "per_layer_GB": round(inc / 1e9, 3), "max_layers_in_180GB": lmax}), flush=True)
        mg.mggcn_part_free(part)
    mg.mggcn_graph_free(g)
