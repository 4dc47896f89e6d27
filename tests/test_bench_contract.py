"""bench.py host-side contract (CPU only): the epoch's SpMM widths and the
L2-line model behind roofline.l2_gather, and the reference arm (the CPU oracle
on a bounded sample) printing one JSON line with the driver's keys."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def test_spmm_widths_follow_the_order_rule():
    import bench
    # Reddit-shaped: every layer GeMM-first (d_l >= d_{l+1}, C10): forward + backward SpMM per layer
    assert sorted(bench.spmm_widths([602, 256, 256, 41])) == [41, 41, 256, 256, 256, 256]
    # Products / Proteins-shaped: SpMM-first layer 0 (forward T0 only, backward skipped, C11)
    assert sorted(bench.spmm_widths([100, 256, 256, 47])) == [47, 47, 100, 256, 256]
    assert sorted(bench.spmm_widths([8, 128, 128, 112])) == [8, 112, 112, 128, 128]


@pytest.mark.parametrize("width,lines", [(256, 8), (128, 4), (41, 2), (48, 2), (100, 4), (8, 1), (602, 19)])
def test_line_bytes(width, lines):
    import bench
    assert bench.line_bytes(width) == pytest.approx(128 * lines, rel=0.2)


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload", "cora",
                        "--steps", "2", "--warmup", "1", "--oracle-rows", "300"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "impl", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["higher_is_better"] is False and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


def test_graph_stats_tile_spread_matches_brute_force():
    """bench.graph_stats: the P x P tile histogram of the permuted partition p(i) = floor(i n / P)
    equals a brute-force assignment by searching the partition boundaries."""
    import numpy as np
    import bench
    import gen
    n = 1003
    rp, col = gen.rmat_csr(n, 20000, 7)
    perm = np.random.default_rng(1).permutation(n).astype(np.int64)
    st = bench.graph_stats(n, rp, col, perm)
    deg = np.diff(rp)
    assert st["deg_max"] == deg.max() and abs(st["deg_mean"] - deg.mean()) < 1e-12
    pu, pv = np.repeat(perm, deg), perm[col]
    for P in (2, 4, 8):
        bnd = (np.arange(P + 1) * n) // P
        bu = np.searchsorted(bnd, pu, side="right") - 1
        bv = np.searchsorted(bnd, pv, side="right") - 1
        c = np.bincount(bu * P + bv, minlength=P * P)
        assert abs(st["tile_nnz_max_over_mean"][P] - c.max() / c.mean()) < 1e-12


def test_timeline_summary_exposed_comm_and_bandwidth():
    """bench.timeline_summary (host logic of the per-stage timeline, Fig. 6 / 8): exposed comm is the
    comm-stream busy time not covered by compute-stream ops; bcast GB/s from the block's bytes."""
    import bench
    tl = [dict(cls="spmm", spmm=0, stage=-1, rank=0, stream=0, t0=0.0, t1=1.0),
          dict(cls="bcast", spmm=0, stage=1, rank=-1, stream=1, t0=0.5, t1=1.5),
          dict(cls="bcast", spmm=0, stage=0, rank=-1, stream=1, t0=1.5, t1=1.6),   # own block (sent)
          dict(cls="spmm", spmm=0, stage=1, rank=0, stream=0, t0=1.6, t1=2.0),
          dict(cls="gemm", spmm=-1, stage=-1, rank=-1, stream=0, t0=2.0, t1=2.5)]
    s = bench.timeline_summary(tl, (8, 4, 2), [0, 1000, 2000], 0)
    assert abs(s["epoch_span_ms"] - 2.5) < 1e-12
    assert abs(s["compute_busy_ms"] - 1.9) < 1e-12
    assert abs(s["comm_busy_ms"] - 1.1) < 1e-12
    assert abs(s["exposed_comm_ms"] - 0.6) < 1e-12          # (1.0..1.5) and (1.5..1.6)
    assert s["bcast_records"] == 1                           # received blocks only
    assert abs(s["bcast_GBps_median"] - 1000 * 4 * 4 / 1e-3 / 1e9) < 1e-9
    assert s["per_spmm"]["0"]["compute_launches"] == 2 and s["per_spmm"]["0"]["width"] == 4


def test_dense_summary_flops_and_roofline():
    """bench.dense_summary: issued MMA work = blocks x 128 x 32 x N x 2 x 3 pieces per SpMM of the
    epoch (N = width rounded up to 16 per 256-column window), and the tensor roofline divides it
    by the dense kernels' live time."""
    import bench
    st = {"blocks": 1000, "block_entries": 600000, "entries": 1000000, "row_groups": 10, "chunks": 50}
    d = bench.dense_summary(st, [602, 256, 256, 41], dense_ms=1.0, bf16_peak=1000.0)
    per_block = 128 * 32 * 2 * 3
    want = 1000 * per_block * (4 * 256 + 2 * 48)        # widths 256 x 4, 41 -> 48 x 2
    assert d["mma_tflop_per_epoch"] == pytest.approx(want / 1e12)
    assert d["entry_frac"] == pytest.approx(0.6)
    assert d["roofline"]["achieved"] == pytest.approx(want / 1e-3 / 1e12)
    assert d["roofline"]["frac"] == pytest.approx(d["roofline"]["achieved"] / 1000.0)
    # widths above 256 run in 256-column windows: 600 -> 256 + 256 + 96
    d2 = bench.dense_summary(st, [600, 600], dense_ms=0.0)
    assert d2["mma_tflop_per_epoch"] == pytest.approx(1000 * per_block * 2 * (256 + 256 + 96) / 1e12)
    assert "roofline" not in d2
    assert bench.dense_summary({"blocks": 0}, [8, 8])["blocks"] == 0


def test_l2_gather_counts_only_gathered_entries():
    """roofline.l2_gather: the entries of the dense blocks are not gathered, so the L2-line model
    scales with the gathered (residual) share."""
    import bench
    work = {"spmm_gather_bytes": 4.0 * 1e6 * sum(bench.spmm_widths([602, 256, 256, 41]))}
    full = bench.l2_gather_roofline([602, 256, 256, 41], work, 1.0)
    part = bench.l2_gather_roofline([602, 256, 256, 41], work, 1.0, gathered_frac=0.25)
    assert part["line_bytes_per_epoch"] == pytest.approx(0.25 * full["line_bytes_per_epoch"])
