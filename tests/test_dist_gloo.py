"""World-size-2 gloo test of the multi-process host path (CPU only): the NCCL
unique-id exchange, per-rank partitions that agree with each other and,
concatenated over ranks, with the oracle's tiles, and the
local-row selection used to feed mggcn_forward."""
import os
import socket
import subprocess
import sys
import textwrap

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WORKER = textwrap.dedent(r'''
import os, sys, pickle
sys.path.insert(0, os.environ["ROOT"])
import numpy as np
import torch.distributed as dist
import gen
import paper_conf_icpp_balinsc22_b200 as mg
from paper_conf_icpp_balinsc22_b200.dist import share_nccl_id, local_rows, max_over_ranks
dist.init_process_group("gloo", init_method="env://")
rank, P = dist.get_rank(), dist.get_world_size()
nid = share_nccl_id(dist, lambda: bytes(range(128)))     # same exchange bench.py runs with mggcn_nccl_unique_id
n, m, seed = 1500, 20000, 7
rp, col = gen.rmat_csr(n, m, 3)
g = mg.mggcn_load_csr(n, rp, col)
part = mg.mggcn_partition(g, P, rank, seed)
info = mg.mggcn_part_info(part)
tiles = {d: [mg.mggcn_part_export_tile(part, d, j) for j in range(P)] for d in (0, 1)}
X = gen.features(n, 5, 11)
Xl = local_rows(info["perm"], info["p"], rank, X)
t = max_over_ranks(dist, 1.0 + rank)
out = {"rank": rank, "id": nid, "perm": info["perm"], "p": info["p"], "tiles": tiles, "Xl": Xl, "tmax": t}
objs = [None] * P
dist.all_gather_object(objs, out)
if rank == 0:
    pickle.dump(objs, open(os.environ["OUT"], "wb"))
dist.destroy_process_group()
''')


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def test_two_rank_host_path(tmp_path):
    import pickle
    import build_mggcn
    build_mggcn.build()
    import gen
    import oracle
    script = tmp_path / "worker.py"
    script.write_text(WORKER)
    out = tmp_path / "out.pkl"
    port = _free_port()
    procs = []
    for r in range(2):
        env = dict(os.environ, ROOT=ROOT, OUT=str(out), MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port),
                   RANK=str(r), WORLD_SIZE="2")
        procs.append(subprocess.Popen([sys.executable, str(script)], env=env))
    for p in procs:
        assert p.wait(timeout=300) == 0
    objs = pickle.load(open(out, "rb"))
    a, b = objs
    assert a["id"] == b["id"] == bytes(range(128))
    assert np.array_equal(a["perm"], b["perm"]) and np.array_equal(a["p"], b["p"])
    assert a["tmax"] == b["tmax"] == 2.0
    rp, col = gen.rmat_csr(1500, 20000, 3)
    pg = oracle.permute_graph(1500, rp, col, None, seed=7)
    for o in objs:
        t = oracle.tiles(pg, 2, o["rank"])
        for d, name in ((0, "F"), (1, "B")):
            for j in range(2):
                lrp, lcol, lval = o["tiles"][d][j]
                orp, ocol, oval = t[name][j]
                assert np.array_equal(lrp, orp) and np.array_equal(lcol, ocol)
                assert np.array_equal(lval.view(np.uint32), oval.view(np.uint32))
    X = gen.features(1500, 5, 11)
    Xp = np.empty_like(X)
    Xp[a["perm"]] = X
    assert np.array_equal(np.concatenate([a["Xl"], b["Xl"]]), Xp)


WORKER15 = textwrap.dedent(r'''
import os, sys, pickle
sys.path.insert(0, os.environ["ROOT"])
import numpy as np
import torch.distributed as dist
import gen
import paper_conf_icpp_balinsc22_b200 as mg
from paper_conf_icpp_balinsc22_b200.dist import share_nccl_id, local_rows
dist.init_process_group("gloo", init_method="env://")
g_rank, P = dist.get_rank(), dist.get_world_size()
Pb = P // 2
i, rep = g_rank % Pb, g_rank // Pb                       # rank (i, r) = r * P' + i (MGGCN_F_REPL2)
nid = share_nccl_id(dist, lambda: bytes(range(128)))
n, m, seed = 1500, 20000, 7
rp, col = gen.rmat_csr(n, m, 3)
g = mg.mggcn_load_csr(n, rp, col)
part = mg.mggcn_partition(g, Pb, i, seed)
info = mg.mggcn_part_info(part)
flags = mg.MGGCN_F_REPL2 | (mg.MGGCN_F_REPLICA1 if rep else 0)
ws = mg.mggcn_workspace_bytes([part], (5, 8, 3), flags)
tiles = {d: [mg.mggcn_part_export_tile(part, d, j) for j in range(Pb)] for d in (0, 1)}
Xl = local_rows(info["perm"], info["p"], i, gen.features(n, 5, 11))
out = {"g": g_rank, "i": i, "rep": rep, "id": nid, "perm": info["perm"], "tiles": tiles, "Xl": Xl, "ws": ws}
objs = [None] * P
dist.all_gather_object(objs, out)
if g_rank == 0:
    pickle.dump(objs, open(os.environ["OUT"], "wb"))
dist.destroy_process_group()
''')


def test_four_rank_15d_host_path(tmp_path):
    """1.5D (c = 2) over 4 processes: ranks (i, r) = r * 2 + i share one id, the two
    replicas of a row block build bit-identical tiles and input rows and the same
    workspace plan, and the blocks of one replica cover X' exactly once."""
    import pickle
    import build_mggcn
    build_mggcn.build()
    import gen
    script = tmp_path / "worker15.py"
    script.write_text(WORKER15)
    out = tmp_path / "out.pkl"
    port = _free_port()
    procs = []
    for r in range(4):
        env = dict(os.environ, ROOT=ROOT, OUT=str(out), MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port),
                   RANK=str(r), WORLD_SIZE="4")
        procs.append(subprocess.Popen([sys.executable, str(script)], env=env))
    for p in procs:
        assert p.wait(timeout=300) == 0
    objs = sorted(pickle.load(open(out, "rb")), key=lambda o: o["g"])
    assert all(o["id"] == bytes(range(128)) for o in objs)
    assert [(o["i"], o["rep"]) for o in objs] == [(0, 0), (1, 0), (0, 1), (1, 1)]
    for i in range(2):
        a, b = objs[i], objs[2 + i]
        assert a["ws"] == b["ws"]
        assert np.array_equal(a["Xl"], b["Xl"])
        for d in (0, 1):
            for ta, tb in zip(a["tiles"][d], b["tiles"][d]):
                for x, y in zip(ta, tb):
                    assert np.array_equal(np.asarray(x).view(np.uint8), np.asarray(y).view(np.uint8))
    X = gen.features(1500, 5, 11)
    Xp = np.empty_like(X)
    Xp[objs[0]["perm"]] = X
    assert np.array_equal(np.concatenate([objs[0]["Xl"], objs[1]["Xl"]]), Xp)
