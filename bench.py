"""Benchmark: full-batch GCN epoch time on B200 (BASELINE.json metric
"full-batch GCN epoch ms at 1/2/4/8 B200; SpMM HBM GB/s vs peak").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload reddit] [--impl mggcn|reference]

A step is one full epoch of the hot path (forward over all layers with the
P-stage SpMM, softmax-CE, backward, W_G all-reduce, Adam) on synthetic
R-MAT inputs shaped like BASELINE.json's config (default configs[1],
Reddit-shaped, which fits one GPU).  Rank 0 prints ONE JSON line.

For N > 1 launch with torchrun (one rank per GPU, NCCL over NVLink); the
library creates its own NCCL communicator from a unique id shared through
torch.distributed.  --impl reference times the CPU oracle (the tier's
reference arm) on a bounded row sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gen  # noqa: E402

METRIC = "full-batch GCN epoch ms"
UNIT = "ms"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=int(os.environ.get("WORLD_SIZE", "1")))
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="reddit", choices=sorted(gen.WORKLOADS))
    ap.add_argument("--impl", default="mggcn", choices=["mggcn", "reference"])
    ap.add_argument("--no-overlap", action="store_true")
    ap.add_argument("--comm", default="nccl", choices=["nccl", "ipc"],
                    help="N > 1 exchange backend: the library's NCCL communicator, or MGGCN_F_IPC "
                         "(copy-engine pulls from CUDA-IPC-mapped peer workspaces)")
    ap.add_argument("--replicas", type=int, default=1, choices=[1, 2],
                    help="2 = 1.5D partitioning (MGGCN_F_REPL2, SURVEY NEXT-4): N/2 row blocks, each held by two "
                         "ranks that split the broadcast stages and sum their partials; N must be a multiple of 4")
    ap.add_argument("--tf32x1", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-exposed", action="store_true", help="skip the N > 1 NO_BCAST exposed-comm ablation")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cache-l0", action="store_true",
                    help="skip the extra MGGCN_F_CACHE_L0 timing (reported under 'cache_l0', never the headline)")
    ap.add_argument("--oracle-rows", type=int, default=0, help="row sample of the oracle leg (0 = auto)")
    ap.add_argument("--graph", action="store_true",
                    help="N > 1: also take the headline from captured-epoch replays (NCCL collectives inside the "
                         "graph; default for N = 1 only, since multi-GPU capture is unverified on one-GPU boxes)")
    ap.add_argument("--eager", action="store_true",
                    help="headline from eager forward/backward/step calls instead of replays of the captured "
                         "epoch (mggcn_epoch_capture); the eager loop is timed either way (profile breakdown)")
    return ap.parse_args()


def workload_desc(w, P):
    return {"workload": f"{w.name}-shaped R-MAT (Graph500 a,b,c,d = .57,.19,.19,.05; symmetric, duplicates kept)",
            "n": w.n, "nnz": w.m, "dims": list(w.dims), "layers": len(w.dims) - 1, "P": P,
            "perm_seed": w.perm_seed, "graph_seed": w.seed_G, "partition": "1D row, P-stage broadcast (BC1/BC2)",
            "l2": "no flush: every epoch streams inputs larger than L2 (features, CSR, activations)"}


def graph_stats(n, rp, col, perm):
    """Realised power-law stress of the synthetic graph: degree max / mean, and the
    spread of non-zeros over the P x P tiles of the permuted 1D partition (max / mean) at P = 2, 4, 8."""
    deg = np.diff(rp)
    out = {"deg_max": int(deg.max()), "deg_mean": float(deg.mean()),
           "deg_max_over_mean": float(deg.max() / max(deg.mean(), 1e-30)), "tile_nnz_max_over_mean": {}}
    pu = np.repeat(perm, deg)               # new id of each entry's row
    pv = perm[col]                          # new id of each entry's column
    for P in (2, 4, 8):
        if n < P:
            continue
        bu = (pu * P) // n                  # block of new id x: largest i with floor(i n / P) <= x
        bv = (pv * P) // n
        # p(i) = floor(i n / P): x is in block i iff p(i) <= x < p(i+1); (x P) // n can be one low
        # when i n / P is fractional, so correct it against the exact boundaries
        bnd = (np.arange(P + 1, dtype=np.int64) * n) // P
        bu = np.where(pu >= bnd[np.minimum(bu + 1, P)], bu + 1, bu)
        bv = np.where(pv >= bnd[np.minimum(bv + 1, P)], bv + 1, bv)
        cnt = np.bincount(bu * P + bv, minlength=P * P)
        out["tile_nnz_max_over_mean"][P] = float(cnt.max() / max(cnt.mean(), 1e-30))
    return out


# ------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.f = tempfile.NamedTemporaryFile(mode="w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "100"], stdout=self.f,
                                      stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        with open(self.f.name) as fh:
            for line in fh:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) >= 9:
                    rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows),
                "power_w_max": max(float(r[3]) for r in rows if r[3].replace(".", "").isdigit())
                if any(r[3].replace(".", "").isdigit() for r in rows) else None}


# ------------------------------------------------------- oracle (CPU) leg
_ORACLE_CACHE = {}


def host_info():
    """CPU model and core count of the host the oracle runs on (SURVEY §8(d) "Oracle timing")."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except Exception:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count(), "affinity_cores": len(os.sched_getaffinity(0))}


class pinned_one_core:
    """Run the oracle single-threaded on ONE core (os.sched_setaffinity), restoring the mask after."""

    def __enter__(self):
        self.old = os.sched_getaffinity(0)
        self.core = min(self.old)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.old)


def oracle_calibration(workload):
    """Full single-core oracle epoch vs the row-sampled estimate, measured once on one host by
    scripts/calibrate_oracle.py (profiles/r02_oracle_calibration.json); None if absent."""
    path = os.path.join(ROOT, "profiles", "r02_oracle_calibration.json")
    try:
        return json.load(open(path)).get(workload)
    except Exception:
        return None


def oracle_epoch_sample(w, rp, col, rows_per_step, seed=0):
    """Time the CPU oracle's ops for ONE epoch of workload `w` restricted to a
    random sample of `rows_per_step` output rows (every SpMM, GEMM and the CE
    of the epoch, in the paper's order, Eq. 5-11); returns (estimated
    full-epoch ms, wall seconds, R).  Row-proportional work is scaled by n/R;
    Adam runs on the full weights."""
    import oracle
    n, L, dims = w.n, len(w.dims) - 1, w.dims
    R = min(rows_per_step, n)
    rows = np.sort(np.random.default_rng(seed).choice(n, R, replace=False))
    key = (w.name, id(rp))
    if key not in _ORACLE_CACHE:
        # a symmetric graph: rows of Â^T have the pattern of A's rows (values 1/deg)
        _, ahat = oracle.normalise(n, rp, col)
        csr = oracle.CSR(np.asarray(rp, np.int64), np.asarray(col, np.int64), ahat)
        B = gen.features(n, max(dims), 12345)      # dense operand rows (values irrelevant for timing)
        _ORACLE_CACHE.clear()
        _ORACLE_CACHE[key] = (csr, B)
    csr, B = _ORACLE_CACHE[key]
    Ws = [gen.glorot(dims[l], dims[l + 1], w.seed_W + l) for l in range(L)]
    y = gen.labels(R, dims[-1], 3)
    cols = lambda d: np.ascontiguousarray(B[:, :d])
    rws = lambda d: np.ascontiguousarray(B[rows, :d])
    wall0 = time.perf_counter()
    Z = None
    for l in range(L):                               # forward (Eq. 5-7, §4.4 order)
        if oracle.spmm_first(dims[l], dims[l + 1]):
            Z = oracle.gemm(oracle.spmm(csr, cols(dims[l]), rows=rows), Ws[l])
        else:
            oracle.gemm(rws(dims[l]), Ws[l])
            Z = oracle.spmm(csr, cols(dims[l + 1]), rows=rows)
        Z = oracle.relu(Z) if l < L - 1 else Z
    oracle.softmax_ce(np.ascontiguousarray(Z), y, R)
    for l in range(L - 1, -1, -1):                   # backward (Eq. 8-11)
        if oracle.spmm_first(dims[l], dims[l + 1]):
            oracle.gemm(rws(dims[l]), rws(dims[l + 1]), transA=True)
        else:
            HWG = oracle.spmm(csr, cols(dims[l + 1]), rows=rows)
            oracle.gemm(rws(dims[l]), HWG, transA=True)
            if l > 0:
                oracle.gemm(HWG, Ws[l], transB=True)
    t_row = time.perf_counter() - wall0
    t = time.perf_counter()
    for l in range(L):                               # Adam, full size
        W = Ws[l].copy()
        oracle.adam(W, np.ascontiguousarray(W * 0.01), np.zeros_like(W), np.zeros_like(W), 1)
    t_fixed = time.perf_counter() - t
    return (t_row * (n / R) + t_fixed) * 1e3, time.perf_counter() - wall0, R


# Measured ceiling of the SpMM's real bound: uniform random 512-B row gathers
# (LDG.128, 16 rows in flight per lane) from an L2-resident 29 MB table on this
# B200 (bench_micro/dsmem_gather.cu, mode 0, x = 0; profiles/r01_dsmem_gather.jsonl).
L2_GATHER_PEAK_GBPS = 19480.5


def _git_blob_sha(path):
    import hashlib
    try:
        data = open(path, "rb").read()
    except Exception:
        return None
    return hashlib.sha1(b"blob %d\0" % len(data) + data).hexdigest()


def library_sha256():
    import hashlib
    try:
        return hashlib.sha256(open(os.path.join(ROOT, "paper_conf_icpp_balinsc22_b200", "libmggcn.so"),
                                   "rb").read()).hexdigest()[:16]
    except Exception:
        return None


def stored_traffic(workload, P):
    """roofline.traffic: DRAM bytes per SpMM launch from one ncu --set full capture
    (scripts/profile_round.sh + scripts/summarize_profiles.py), with the build it was taken on."""
    path = os.path.join(ROOT, "profiles", f"spmm_traffic_{workload}_P{P}.json")
    if not os.path.exists(path):
        return None, None
    try:
        d = json.load(open(path))
    except Exception:
        return None, None
    cur = library_sha256()
    return d.get("dram_bytes_per_launch"), {
        "file": os.path.relpath(path, ROOT), "tag": d.get("tag"), "git_sha": d.get("git_sha"),
        "so_sha256": d.get("so_sha256"), "current_so_sha256": cur,
        "same_build": (d.get("so_sha256") == cur) if d.get("so_sha256") else None}


def dense_summary(st, dims, dense_ms=0.0, bf16_peak=1352.7):
    """The dense-block part of the SpMM (DESIGN §6 "Dense blocks"): blocks, the share of the
    coalesced entries they cover, and the tensor work they issue per epoch (128 x 32 x N x 2 flops
    per block per bf16 piece, N = the SpMM width rounded up to 16 per 256-column window)."""
    if not st or not st.get("blocks"):
        return {"blocks": 0, "note": "no tile passed the dense rules (MGGCN_DENSE_THR / _MINFRAC / _MIN_ROWS)"}
    pieces = int(os.environ.get("MGGCN_DENSE_PIECES", "3")) if os.environ.get("MGGCN_DENSE_PIECES") == "2" else 3
    flops = 0.0
    for wdt in spmm_widths(dims):
        n_pad = sum((min(256, wdt - c0) + 15) // 16 * 16 for c0 in range(0, wdt, 256))
        flops += st["blocks"] * 128 * 32 * n_pad * 2 * pieces
    out = {"blocks": st["blocks"], "block_entries": st["block_entries"], "entries": st["entries"],
           "entry_frac": st["block_entries"] / max(st["entries"], 1), "row_groups": st["row_groups"],
           "chunks": st["chunks"], "pieces": pieces, "mma_tflop_per_epoch": flops / 1e12,
           "thr": os.environ.get("MGGCN_DENSE_THR", "default 0.04")}
    if dense_ms > 0:
        ach = flops / (dense_ms * 1e-3) / 1e12
        out["roofline"] = {"bound": "tensor", "achieved": ach, "peak": bf16_peak, "unit": "TFLOP/s",
                           "frac": ach / bf16_peak, "ms_per_epoch": dense_ms,
                           "how": "issued bf16 MMA work (128 x 32 x N x 2 flops x pieces per block) / the dense "
                                  "kernels' time (library CUDA events around B images + blocks + fix-up, profile "
                                  "class 'dense'), against MEASURED_PEAKS bf16 sustained (timed inside the epoch)"}
    return out


def spmm_widths(dims):
    """Widths of the SpMMs of one epoch (§4.4 order rule C10, first-layer skip C11)."""
    ws = []
    for l in range(len(dims) - 1):
        if dims[l] < dims[l + 1]:          # SpMM-first (layer 0 only): forward T0 = A'^T X; no backward SpMM
            ws.append(dims[l])
        else:                              # GeMM-first: forward A'^T HW and backward A' AHW_G
            ws += [dims[l + 1], dims[l + 1]]
    return ws


def line_bytes(width):
    """Bytes of 128-B L2 lines one gathered row touches: the kernel reads ceil(width/4) float4
    of a row whose stride is ld = round_up(width, 8) floats (window of <= 128 floats when the
    library splits the width), averaged over the row start offsets mod 128 B."""
    tot = 0
    c0 = 0
    while c0 < width:
        w = min(128 if width > 128 else width, width - c0)
        ld_b = ((width + 7) // 8 * 8) * 4
        rd = (w + 3) // 4 * 16
        offs = sorted({(r * ld_b + c0 * 4) % 128 for r in range(128)})
        tot += sum(((o + rd + 127) // 128) * 128 for o in offs) / len(offs)
        c0 += w
    return tot


def l2_gather_roofline(dims, work, spmm_ms_per_epoch, cache=False, gathered_frac=1.0):
    ws = spmm_widths(dims)
    # coalesced non-zeros per SpMM (all ranks' tiles) that the CSR kernel gathers: the entries of
    # the dense blocks run on the tensor cores instead
    nnz = work["spmm_gather_bytes"] / (4.0 * sum(ws)) * gathered_frac
    lb = nnz * sum(line_bytes(x) for x in ws)
    ach = lb / (spmm_ms_per_epoch * 1e-3) / 1e9 if spmm_ms_per_epoch > 0 else 0.0
    return {"bound": "l2 (SM<-L2 line rate of random row gathers)", "achieved": ach, "peak": L2_GATHER_PEAK_GBPS,
            "unit": "GB/s", "frac": ach / L2_GATHER_PEAK_GBPS, "line_bytes_per_epoch": lb,
            "peak_source": "bench_micro/dsmem_gather.cu: uniform 512-B row gathers from an L2-resident table "
                           "(profiles/r01_dsmem_gather.jsonl)",
            "peak_source_blob_sha": _git_blob_sha(os.path.join(ROOT, "bench_micro", "dsmem_gather.cu"))}


def _union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def _measure(iv):
    return sum(b - a for a, b in iv)


def _intersect(u, v):
    i = j = 0
    tot = 0.0
    while i < len(u) and j < len(v):
        a, b = max(u[i][0], v[j][0]), min(u[i][1], v[j][1])
        if b > a:
            tot += b - a
        if u[i][1] < v[j][1]:
            i += 1
        else:
            j += 1
    return tot


def timeline_summary(tl, dims, p, rank):
    """Per-stage comm / compute timeline of one epoch (MGGCN_F_TIMELINE; the paper's Fig. 6 / 8,
    P:1372-1403): busy time per stream, the comm time not covered by any compute
    op (exposed), and broadcast GB/s per received block."""
    L = len(dims) - 1
    fwd = [dims[l] if dims[l] < dims[l + 1] else dims[l + 1] for l in range(L)]
    bwd = [dims[l + 1] for l in range(L - 1, -1, -1) if dims[l] >= dims[l + 1]]
    widths = fwd + bwd
    comp = [(r["t0"], r["t1"]) for r in tl if r["stream"] == 0]
    comm = [(r["t0"], r["t1"]) for r in tl if r["stream"] == 1]
    if not comp:
        return None
    t0 = min(a for a, _ in comp + comm)
    t1 = max(b for _, b in comp + comm)
    uc, um = _union(comp), _union(comm)
    exposed = _measure(um) - _intersect(um, uc)
    gbps = []
    for r in tl:
        if r["stream"] == 1 and r["cls"] == "bcast" and 0 <= r["spmm"] < len(widths) and r["stage"] >= 0 \
                and r["stage"] != rank and r["t1"] > r["t0"]:
            rows = int(p[r["stage"] + 1] - p[r["stage"]])
            gbps.append(rows * widths[r["spmm"]] * 4 / ((r["t1"] - r["t0"]) * 1e-3) / 1e9)
    per = {}
    for r in tl:
        if r["spmm"] < 0:
            continue
        d = per.setdefault(r["spmm"], {"width": widths[r["spmm"]] if r["spmm"] < len(widths) else None,
                                       "compute_launches": 0, "compute_ms": 0.0, "comm_ops": 0, "comm_ms": 0.0,
                                       "dense_ms": 0.0})
        if r["cls"] == "dense":          # nested inside its stage's spmm record
            d["dense_ms"] += r["t1"] - r["t0"]
        elif r["stream"] == 0:
            d["compute_launches"] += 1
            d["compute_ms"] += r["t1"] - r["t0"]
        else:
            d["comm_ops"] += 1
            d["comm_ms"] += r["t1"] - r["t0"]
    return {"epoch_span_ms": t1 - t0, "compute_busy_ms": _measure(uc), "comm_busy_ms": _measure(um),
            "exposed_comm_ms": exposed, "exposed_comm_frac": exposed / (t1 - t0) if t1 > t0 else None,
            "bcast_GBps_median": statistics.median(gbps) if gbps else None, "bcast_records": len(gbps),
            "per_spmm": {str(k): {kk: (round(vv, 4) if isinstance(vv, float) else vv) for kk, vv in v.items()}
                         for k, v in sorted(per.items())},
            "how": "one eager epoch with MGGCN_F_TIMELINE (CUDA event pair per op on the stream it runs on; the "
                   "timed epochs run without it); exposed = comm-stream busy time not covered by any compute-stream "
                   "op; bcast GB/s = received block bytes / broadcast duration"}


def auto_rows(w):
    # about 3 s of single-core oracle work per sampled epoch
    per_row = (w.m / w.n) * sum(w.dims) * 2 + 3 * sum(w.dims[l] * w.dims[l + 1] for l in range(len(w.dims) - 1))
    return int(max(200, min(w.n, 1.5e9 / per_row)))


def run_reference(args):
    """Reference arm of this tier: the CPU oracle, as it stands, on host cores."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    w = gen.WORKLOADS[args.workload]
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    R = args.oracle_rows or auto_rows(w)
    vals, walls = [], []
    with pinned_one_core():
        for s in range(args.warmup + args.steps):
            est, wall, _ = oracle_epoch_sample(w, rp, col, R, seed=s)
            if s >= args.warmup:
                vals.append(est)
                walls.append(wall)
    raw = statistics.median(vals)
    cal = oracle_calibration(w.name)
    value = raw * cal["ratio"] if cal else raw
    sample = (f"{R} random output rows of every SpMM/GEMM/CE op of one epoch (n = {w.n}), scaled by n/R; Adam full; "
              f"one pinned core" + ("; x calibration ratio full/sampled from profiles/r02_oracle_calibration.json"
                                   if cal else "; uncalibrated"))
    line = {"metric": METRIC, "value": value, "unit": UNIT, "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": statistics.median(walls) * 1e3,
            "higher_is_better": False, "scaling": "strong", "vs_baseline": None, "dtype": "f32 storage, f64 accumulate",
            "data": "synthetic", "config": workload_desc(w, args.gpus),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                             "estimated": True, "rows_sampled": R, "sampled_estimate_ms": raw, "calibration": cal,
                             "host": host_info()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------ GPU arm
def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_balinsc22_b200 as mg
    from paper_conf_icpp_balinsc22_b200 import GCN
    from paper_conf_icpp_balinsc22_b200.dist import ipc_exchange, max_over_ranks, share_nccl_id

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    P = world
    torch.cuda.set_device(local % torch.cuda.device_count())   # (IPC ranks may share a GPU in tests)
    if world > 1:
        # control plane only (NCCL unique id, barriers, max over ranks): gloo.  The data
        # path's broadcasts and all-reduces run on the library's own NCCL communicator.
        dist.init_process_group("gloo")
    w = gen.WORKLOADS[args.workload]

    t0 = time.perf_counter()
    rp, col = gen.rmat_csr(w.n, w.m, w.seed_G)
    X = gen.features(w.n, w.dims[0], w.seed_X)
    y = gen.labels(w.n, w.dims[-1], w.seed_y)
    Ws = [gen.glorot(w.dims[l], w.dims[l + 1], w.seed_W + l) for l in range(len(w.dims) - 1)]
    t_gen = time.perf_counter() - t0


    def comm_kw():
        if world == 1:
            return {}
        if args.comm == "ipc":
            return {"comm": "ipc", "ipc_exchange": ipc_exchange(dist)}
        return {"nccl_id": share_nccl_id(dist, mg.mggcn_nccl_unique_id)}
    flags = mg.MGGCN_F_PROFILE | (0 if args.no_overlap else mg.MGGCN_F_OVERLAP)
    if args.tf32x1:
        flags |= mg.MGGCN_F_TF32X1
    t0 = time.perf_counter()
    graph = mg.mggcn_load_csr(w.n, rp, col)
    if args.replicas > 1 and (P % (2 * args.replicas) or args.comm == "ipc"):
        raise SystemExit("--replicas 2 needs N a multiple of 4 and the NCCL backend")
    gm = GCN(w.n, rp, col, None, w.dims, P=P, rank=rank, perm_seed=w.perm_seed, flags=flags, graph=graph,
             replicas=args.replicas, **comm_kw())
    t_setup = time.perf_counter() - t0
    gm.set_weights(Ws)
    Xl = gm.permute_rows(X)
    yl = gm.permute_rows(y)
    del X
    Xd = gm.device_inputs(Xl)          # padded device layout: layer 0 reads it in place
    yd = torch.from_numpy(yl).cuda()
    torch.cuda.synchronize()

    def epoch(Xin, yin, want_loss=False):
        loss = gm.forward(Xin, yin, want_loss=want_loss)
        gm.backward()
        gm.step(lr=0.01)
        return loss

    for _ in range(args.warmup):
        epoch(Xd, yd)
    gm.synchronize()
    gm.profile(reset=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)       # let the sampler start
    launches0 = mg.mggcn_kernel_launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(gm.cs)
    for _ in range(args.steps):
        epoch(Xd, yd)
    ev1.record(gm.cs)
    ev1.synchronize()
    gm.synchronize()
    launches = mg.mggcn_kernel_launch_count() - launches0
    clk = clocks.stop()
    if world > 1:
        dist.barrier()
    ms = ev0.elapsed_time(ev1) / args.steps
    prof = gm.profile(reset=True)
    work = gm.epoch_work()
    work_detail = gm.epoch_work_detail()
    stage_groups = mg.mggcn_stage_groups(gm.m)
    dense_stats = mg.mggcn_dense_stats(gm.m)
    # ---- one extra eager epoch with the per-stage timeline (not timed)
    timeline = None
    try:
        mg.mggcn_get_timeline(gm.m, reset=True)
        mg.mggcn_timeline_enable(gm.m, True)
        epoch(Xd, yd)
        gm.synchronize()
        tl = mg.mggcn_get_timeline(gm.m, reset=True)
        mg.mggcn_timeline_enable(gm.m, False)
        gm.profile(reset=True)
        timeline = timeline_summary(tl, w.dims, gm.p, rank % (P // args.replicas))
    except mg.MggcnError as e:
        timeline = {"error": str(e)}
    ms_eager = max_over_ranks(dist, ms)

    # ---- the same epochs as one CUDA graph each (mggcn_epoch_capture / _replay): identical
    # kernels and stream order, no per-kernel host launch gaps; the headline unless --eager.
    # The graph is captured without the profiling events, so this loop has no per-op events.
    gtime = None
    if not args.eager and args.comm != "ipc" and (world == 1 or args.graph):
        gm.capture_epoch(Xd, yd, lr=0.01)
        gm.replay_epoch(args.warmup)
        gm.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        clocks_g = ClockSampler(local)
        clocks_g.start()
        time.sleep(0.3)
        gl0 = mg.mggcn_kernel_launch_count()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record(gm.cs)
        for _ in range(args.steps):
            gm.replay_epoch(1)
        g1.record(gm.cs)
        g1.synchronize()
        gm.synchronize()
        glaunch = mg.mggcn_kernel_launch_count() - gl0
        clk_g = clocks_g.stop()
        if world > 1:
            dist.barrier()
        gtime = {"ms": max_over_ranks(dist, g0.elapsed_time(g1) / args.steps), "launches": int(glaunch),
                 "clocks": clk_g}
    if gtime is not None:
        ms_max, launches, clk = gtime["ms"], gtime["launches"], gtime["clocks"]
    else:
        ms_max = ms_eager

    # ---- end to end: host (pinned) inputs through the C ABI, loss read back every step.
    # Each step's X, y are copied host -> device inside the timed region; the copy of
    # step k+1 is enqueued (mggcn_prefetch, library copy stream) while step k computes.
    e2e = None
    if not args.no_e2e:
        # pinned host X in the library's padded row layout (d_0 rounded up to 8 floats): the H2D is
        # then one contiguous copy per step, no device-side restaging (mggcn.h, mggcn_forward)
        Xh = torch.zeros((Xl.shape[0], gm.ld0), dtype=torch.float32).pin_memory()
        Xh[:, :Xl.shape[1]] = torch.from_numpy(Xl)
        yh = torch.from_numpy(yl).pin_memory()

        def e2e_steps(k_steps):
            losses = []
            gm.prefetch(Xh, yh)
            for k in range(k_steps):
                gm.forward(None, None, want_loss=False)
                if k + 1 < k_steps:
                    gm.prefetch(Xh, yh)
                gm.backward()
                gm.step(lr=0.01)
                losses.append(gm.loss())          # D2H of the step's loss (synchronising)
            return losses

        e2e_steps(2)
        gm.synchronize()
        if world > 1:
            dist.barrier()
        tw = time.perf_counter()
        e2e_steps(args.steps)
        gm.synchronize()
        e2e_ms = (time.perf_counter() - tw) * 1e3 / args.steps
        e2e = {"value": max_over_ranks(dist, e2e_ms), "unit": UNIT,
               "h2d_bytes_per_step": int(Xh.numel() * 4 + yl.nbytes), "d2h_bytes_per_step": 16,
               "how": "wall clock over K epochs through the C ABI: X (padded rows), y of every step copied from pinned "
                      "host memory (step k+1's copy overlaps step k via mggcn_prefetch), loss read back every step"}
    loss_now = gm.loss()

    # ---- extra (not the headline): layer-0 aggregation cache, SURVEY NEXT-2
    cache_l0 = None
    if not args.no_cache_l0:
        Ws_now = gm.get_weights()
        gm.close()
        del gm
        torch.cuda.empty_cache()
        gc = GCN(w.n, rp, col, None, w.dims, P=P, rank=rank, perm_seed=w.perm_seed,
                 flags=flags | mg.MGGCN_F_CACHE_L0, graph=graph, replicas=args.replicas, **comm_kw())
        gc.set_weights(Ws_now)
        for _ in range(max(args.warmup, 1)):
            gc.forward(Xd, yd, want_loss=False)
            gc.backward()
            gc.step(lr=0.01)
        gc.synchronize()
        if world > 1:
            dist.barrier()
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        c0.record(gc.cs)
        for _ in range(args.steps):
            gc.forward(Xd, yd, want_loss=False)
            gc.backward()
            gc.step(lr=0.01)
        c1.record(gc.cs)
        c1.synchronize()
        cache_l0 = {"value": max_over_ranks(dist, c0.elapsed_time(c1) / args.steps), "unit": UNIT,
                    "note": "MGGCN_F_CACHE_L0: T0 = A'^T X computed once (first forward), layer 0 = T0 W0 and "
                            "W_G0 = T0^T Z_G0 (exact by associativity); removes both layer-0 SpMMs per epoch. "
                            "Opt-in; not the headline value."}
        gm = gc

    # ---- N > 1: exposed communication by ablation (SURVEY §8(d) "How to time it"): the same eager
    # epochs with MGGCN_F_NO_BCAST (timing only: broadcasts skipped, results invalid; the W_G and
    # loss all-reduces still run) give the compute-only time T_c; exposed = (T - T_c) / T.
    exposed = None
    if world > 1 and not args.no_exposed:
        Ws_now = gm.get_weights()
        gm.close()
        del gm
        torch.cuda.empty_cache()
        gn = GCN(w.n, rp, col, None, w.dims, P=P, rank=rank, perm_seed=w.perm_seed,
                 flags=flags | mg.MGGCN_F_NO_BCAST, graph=graph, replicas=args.replicas, **comm_kw())
        gn.set_weights(Ws_now)
        for _ in range(args.warmup):
            gn.forward(Xd, yd, want_loss=False)
            gn.backward()
            gn.step(lr=0.01)
        gn.synchronize()
        dist.barrier()
        torch.cuda.synchronize()
        n0, n1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        n0.record(gn.cs)
        for _ in range(args.steps):
            gn.forward(Xd, yd, want_loss=False)
            gn.backward()
            gn.step(lr=0.01)
        n1.record(gn.cs)
        n1.synchronize()
        gn.synchronize()
        dist.barrier()
        t_c = max_over_ranks(dist, n0.elapsed_time(n1) / args.steps)
        exposed = {"compute_only_ms": t_c, "eager_ms": ms_eager,
                   "frac": max(0.0, (ms_eager - t_c) / ms_eager) if ms_eager > 0 else None,
                   "bcast_bytes_per_rank_per_epoch": work["bcast_bytes"],
                   "nvlink_bound_ms": work["bcast_bytes"] / 900e9 * 1e3,
                   "how": "(eager epoch ms - the same epochs with MGGCN_F_NO_BCAST) / eager epoch ms, max over ranks; "
                          "target < 0.15 (north_star)"}
        gm = gn
    mg.mggcn_graph_free(graph)
    gstats = graph_stats(w.n, rp, col, np.asarray(gm.perm, dtype=np.int64)) if rank == 0 else None

    if rank != 0:
        gm.close()
        if world > 1:
            dist.destroy_process_group()
        return

    peaks = {}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            peaks = json.load(f)
    except Exception:
        pass
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "MEASURED_PEAKS.json hbm_gbs (measured)" if "hbm_gbs" in peaks else "fallback 6.65 TB/s"
    spmm_ms, spmm_n = prof["spmm"]
    spmm_launch_ms = spmm_ms / max(spmm_n, 1)
    launches_per_epoch = spmm_n / args.steps
    wd = work_detail
    # SURVEY §8(d) compulsory bytes: 4 B per non-zero of the tiles as partitioned (pattern-only),
    # rowptr, each gathered row once, each output row once
    bytes_per_launch = wd["spmm_bytes"] / max(launches_per_epoch, 1)
    struct_per_launch = wd["spmm_struct_bytes"] / max(launches_per_epoch, 1)
    achieved = bytes_per_launch / (spmm_launch_ms * 1e-3) / 1e9 if spmm_ms > 0 else 0.0
    gather_gbs = (wd["spmm_gather_bytes"] / max(launches_per_epoch, 1)) / (spmm_launch_ms * 1e-3) / 1e9 \
        if spmm_ms > 0 else 0.0
    traffic, traffic_src = stored_traffic(args.workload, P)
    gathered_frac = 1.0 - (dense_stats["block_entries"] / dense_stats["entries"]
                           if dense_stats.get("entries") else 0.0)
    l2_gather = l2_gather_roofline(w.dims, work, spmm_ms / args.steps, cache=False, gathered_frac=gathered_frac)
    l2_gather["gathered_entry_frac"] = gathered_frac
    l2_gather["note"] = ("line bytes of the gathered (residual) entries over the whole SpMM time, which also "
                         "contains the dense blocks' kernels: a lower bound on the gather kernel's own rate")
    gemm_ms, gemm_n = prof["gemm"]
    # dense TF32 peak = the measured bf16 peak x the nominal tf32 : bf16 ratio (1 : 2); the GEMMs are
    # timed inside a long epoch, so the sustained figure is the denominator of their fraction
    tf32_peak = float(peaks.get("bf16_tflops_sustained", 1352.7)) / 2.0
    tf32_burst = float(peaks.get("bf16_tflops", 1623.0)) / 2.0
    gemm_tflops = wd["gemm_flops"] / (gemm_ms / args.steps * 1e-3) / 1e12 if gemm_ms else None
    mma_passes = 1 if args.tf32x1 else 3            # 3xTF32 issues hi*hi + hi*lo + lo*hi
    # per-epoch roofline (BASELINE.json metric; SURVEY §8(d) "Per-epoch bounds per GPU")
    nvlink = 900.0
    t_spmm = wd["spmm_bytes"] / (hbm * 1e9) * 1e3
    t_gemm = wd["gemm_flops"] / (tf32_burst * 1e12) * 1e3
    t_bc = wd["bcast_bytes"] / (nvlink * 1e9) * 1e3
    hbm_all = wd["spmm_bytes"] + wd["gemm_bytes"] + wd["ce_bytes"] + wd["bcast_bytes"]
    t_tight_hbm = hbm_all / (hbm * 1e9) * 1e3
    official = max(t_spmm, t_gemm, t_bc)
    tight = max(t_tight_hbm, t_gemm, t_bc)
    epoch_roofline = {
        "official_bound_ms": official, "official_frac": official / ms_max,
        "tight_bound_ms": tight, "tight_frac": tight / ms_max,
        "terms_ms": {"spmm_compulsory_over_hbm": t_spmm, "gemm_flops_over_tf32": t_gemm,
                     "bcast_over_nvlink": t_bc, "all_compulsory_hbm_bytes_over_hbm": t_tight_hbm},
        "bytes": {"spmm_compulsory": wd["spmm_bytes"], "gemm_operands": wd["gemm_bytes"], "ce": wd["ce_bytes"],
                  "bcast_recv": wd["bcast_bytes"]},
        "gemm_gflop": wd["gemm_flops"] / 1e9,
        "peaks": {"hbm_GBps": hbm, "tf32_TFLOPs": tf32_burst, "nvlink_GBps": nvlink},
        "how": "official = max(SpMM compulsory bytes / HBM, GEMM flops / dense TF32, broadcast bytes / NVLink) "
               "(BASELINE.json north_star); tight = max(all compulsory HBM bytes incl. GEMM operands, CE and "
               "broadcast writes / HBM, the other two); frac = bound / measured epoch ms (this line's value)"}
    line = {
        "metric": METRIC, "value": ms_max, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max, "higher_is_better": False, "scaling": "strong",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": workload_desc(w, P),
        "run": {"overlap": not args.no_overlap, "gemm": "tf32x1" if args.tf32x1 else "3xTF32 (tcgen05)",
                "stage_groups": stage_groups,
                "comm": (args.comm if P > 1 else "none"),
                "parallelism": (f"dp{P} (1D row partition)" if args.replicas == 1 else
                                f"dp{P} (1.5D: {P // 2} row blocks x 2 replicas)")},
        "timing": ("K replays of the captured epoch (mggcn_epoch_replay), CUDA events on the compute stream"
                   if gtime is not None else "K eager forward/backward/step epochs, CUDA events on the compute stream"),
        "eager_ms": ms_eager,
        "e2e": e2e,
        "gpu_launches": int(launches),
        "clocks": clk,
        "roofline": {"bound": "hbm", "kernel": "SpMM stage (F2/B1): dense_tile_kernel (tcgen05 bf16x3 blocks) + "
                                               "spmm_stage_kernel (CSR gather of the residual entries)",
                     "achieved": achieved, "peak": hbm, "unit": "GB/s", "frac": achieved / hbm,
                     "traffic": traffic, "traffic_source": traffic_src, "peak_source": peak_src,
                     "algorithmic_bytes_per_launch": bytes_per_launch,
                     "struct_bytes_per_launch": struct_per_launch,
                     "launch_ms": spmm_launch_ms, "launches_per_epoch": launches_per_epoch,
                     "gather_model_GBps": gather_gbs,
                     "note": "achieved = SURVEY §8(d) compulsory bytes (4 B per non-zero of the partitioned "
                             "tiles, rowptr, each gathered and each output row once) / measured mean launch time "
                             "(CUDA events on the compute stream); struct_bytes_per_launch = the same with the "
                             "device tiles' coalesced (index + multiplicity) entries; gather_model_GBps = "
                             "coalesced nnz * width * 4 B / time; a launch = one SpMM stage (B images + dense "
                             "blocks + their fix-up, the column-window gather kernels + hub fix-up)",
                     "l2_gather": l2_gather},
        "epoch_roofline": epoch_roofline,
        "dense": dense_summary(dense_stats, w.dims, prof.get("dense", (0.0, 0))[0] / args.steps,
                               float(peaks.get("bf16_tflops_sustained", 1352.7))),
        "breakdown_ms_per_epoch": {k: v[0] / args.steps for k, v in prof.items()},
        "gemm": {"tflops": gemm_tflops, "peak_tf32_tflops": tf32_peak, "ms_per_epoch": gemm_ms / args.steps,
                 "frac_model_flops": gemm_tflops / tf32_peak if gemm_tflops else None,
                 "mma_passes": mma_passes,
                 "tensor_frac": gemm_tflops * mma_passes / tf32_peak if gemm_tflops else None,
                 "how": "model flops 2MNK per product / GEMM ms per epoch (CUDA events); tensor_frac counts the "
                        "MMA work actually issued (3 TF32 passes for 3xTF32) against the sustained dense TF32 "
                        "peak (MEASURED_PEAKS bf16 sustained / 2)"},
        "loss_after": loss_now,
        "cache_l0": cache_l0,
        "exposed_comm": exposed,
        "timeline": timeline,
        "graph_stats": gstats,
        "setup_s": {"generate": t_gen, "load_csr+partition+upload": t_setup},
    }
    # ---- CPU baseline: the oracle on a bounded sample (rank 0, N = 1 only)
    if world == 1 and not args.no_cpu_baseline:
        R = args.oracle_rows or auto_rows(w)
        ests = []
        with pinned_one_core():
            for s in range(3):
                est, _, _ = oracle_epoch_sample(w, rp, col, R, seed=s)
                ests.append(est)
        raw = statistics.median(ests)
        cal = oracle_calibration(w.name)
        line["cpu_baseline"] = {"value": raw * cal["ratio"] if cal else raw, "unit": UNIT, "cores": 1, "kind": "oracle",
                                "sample": f"3 x {R} random output rows of every SpMM/GEMM/CE op of one epoch "
                                          f"(n = {w.n}), scaled by n/R; Adam full; one pinned core" +
                                          ("; x calibration ratio (full single-core oracle epoch / sampled estimate, "
                                           "profiles/r02_oracle_calibration.json)" if cal else "; uncalibrated"),
                                "estimated": True, "rows_sampled": R, "sampled_estimate_ms": raw,
                                "calibration": cal, "host": host_info()}
    print(json.dumps(line), flush=True)
    gm.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
