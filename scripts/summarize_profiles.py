"""Summarise the ncu captures of scripts/profile_round.sh into profiles/.

    python scripts/summarize_profiles.py <tag> [workload]

Writes profiles/<tag>_launches.csv (the per-launch gpu__time_duration list of
one epoch, cold-cache and serialised under ncu), profiles/<tag>_summary.md
(per-kernel metrics from the --set full captures) and
profiles/spmm_traffic_<workload>_P1.json (DRAM bytes per SpMM launch, read by
bench.py for roofline.traffic).
"""
import csv
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % of peak"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit %"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor pipe active %"),
    ("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "tcgen05 pipe active % (of active cycles)"),
    ("sm__pipe_tc_cycles_active.min.pct_of_peak_sustained_active", "tcgen05 pipe active %, least busy SM"),
    ("sm__pipe_tc_cycles_active.max.pct_of_peak_sustained_active", "tcgen05 pipe active %, busiest SM"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("smsp__inst_executed.sum", "warp instructions"),
]


def raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    if len(rows) < 3:
        return None
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (u, v) for h, u, v in zip(hdr, units, vals)}, hdr, vals


def to_bytes(u, v):
    v = float(v)
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)


def main():
    tag = sys.argv[1]
    wl = sys.argv[2] if len(sys.argv) > 2 else "reddit"
    os.makedirs(PROF, exist_ok=True)
    lines = [f"# ncu summary `{tag}` — workload {wl}-shaped, P = 1 (`bench.py --steps 1 --warmup 1`)", "",
             "Captured on one B200 with `scripts/profile_round.sh` (`ncu --set full --clock-control none`,"
             " one launch each, cold cache, replayed); times here are ncu's, not bench values.", ""]
    # launch list
    lc = os.path.join(OUT, f"{tag}_launches.csv")
    if os.path.exists(lc):
        shutil.copy(lc, os.path.join(PROF, f"{tag}_launches.csv"))
        rows = list(csv.reader(open(lc)))
        hdr = None
        launches = []
        for r in rows:
            if "Kernel Name" in r:
                hdr = r
                continue
            if hdr and len(r) == len(hdr):
                d = dict(zip(hdr, r))
                launches.append((int(d["ID"]), d["Kernel Name"], float(d["Metric Value"])))
        # the timed epoch (the second of the bench's model, after one warm-up epoch): the launches
        # after the first Adam's weight re-split up to and including the second Adam's
        adam_ids = [i for i, n, _ in launches if "adam_kernel" in n]
        if len(adam_ids) >= 2:
            ep = [(i, n, t) for i, n, t in launches if adam_ids[0] + 3 < i <= adam_ids[1] + 3]
        else:
            ep = launches
        tot = sum(t for _, _, t in ep)
        share = {}
        for _, n, t in ep:
            k = n.split("(")[0].split("::")[-1].split("<")[0]
            share[k] = share.get(k, 0.0) + t
        lines += ["## Per-kernel share of one epoch (ncu launch list, serialised, cold cache)", "",
                  "| kernel | launches | total µs | share |", "|---|---|---|---|"]
        counts = {}
        for _, n, _ in ep:
            k = n.split("(")[0].split("::")[-1].split("<")[0]
            counts[k] = counts.get(k, 0) + 1
        for k, t in sorted(share.items(), key=lambda x: -x[1]):
            lines.append(f"| {k} | {counts[k]} | {t / 1e3:.1f} | {t / tot:.1%} |")
        lines.append(f"| **total** | {len(ep)} | {tot / 1e3:.1f} | 100% |")
        lines.append("")
    traffic = {}
    for name in ("dense_tile", "spmm_wide", "spmm_narrow", "gemm_rows", "gemm_wgrad"):
        rep = os.path.join(OUT, f"{tag}_{name}.ncu-rep")
        if not os.path.exists(rep):
            continue
        shutil.copy(rep, os.path.join(PROF, f"{tag}_{name}.ncu-rep"))
        res = raw(rep)
        if not res:
            continue
        d, hdr, vals = res
        lines += [f"## `{name}`", "", "| metric | value |", "|---|---|"]
        for m, label in METRICS:
            if m in d:
                u, v = d[m]
                lines.append(f"| {label} (`{m}`) | {v} {u} |")
        stalls = []
        for h, (u, v) in d.items():
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    stalls.append((float(v), h.replace("smsp__average_warps_issue_stalled_", "").replace(
                        "_per_issue_active.ratio", "")))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        lines.append("| top stall reasons (cycles / issued inst) | " +
                     ", ".join(f"{s} {v:.2f}" for v, s in stalls[:4]) + " |")
        lines.append("")
        if (name.startswith("spmm") or name == "dense_tile") and "dram__bytes_read.sum" in d:
            traffic[name] = to_bytes(*d["dram__bytes_read.sum"]) + to_bytes(*d["dram__bytes_write.sum"])
            traffic[name + "_ms"] = float(d["gpu__time_duration.sum"][1]) * (
                1e-3 if d["gpu__time_duration.sum"][0] == "us" else 1.0)
    if "spmm_wide" in traffic:
        # an epoch has 4 wide (256) and 2 narrow (41 -> 48) SpMM stages for the Reddit config; a wide
        # stage is 2 column-window launches of 128 floats (spmm.cu launch_spmm), the capture is one window
        nwin = int(os.environ.get("WIDE_WINDOWS", "2" if wl == "reddit" else "1"))
        # a wide stage also runs the dense blocks (one dense_tile_kernel launch, captured separately;
        # the narrow stage's dense launch is not captured, so `narrow` counts its gather only)
        wide = nwin * traffic["spmm_wide"] + traffic.get("dense_tile", 0.0)
        narrow = traffic.get("spmm_narrow", traffic["spmm_wide"])
        avg = (4 * wide + 2 * narrow) / 6 if wl == "reddit" else wide
        import hashlib
        so = os.path.join(ROOT, "paper_conf_icpp_balinsc22_b200", "libmggcn.so")
        so_sha = open(os.path.join(OUT, f"{tag}_so.sha")).read().split()[0][:16] \
            if os.path.exists(os.path.join(OUT, f"{tag}_so.sha")) else hashlib.sha256(open(so, "rb").read()).hexdigest()[:16]
        git_sha = subprocess.run(["git", "-C", ROOT, "rev-parse", "HEAD"], capture_output=True, text=True).stdout.strip()
        json.dump({"workload": wl, "P": 1, "tag": tag, "dram_bytes_per_launch": avg,
                   "so_sha256": so_sha, "git_sha": git_sha,
                   "dram_bytes_wide_launch": wide, "dram_bytes_narrow_launch": narrow,
                   "dram_bytes_dense_tile_launch": traffic.get("dense_tile"),
                   "wide_windows": nwin,
                   "how": "ncu --set full, dram__bytes_read.sum + dram__bytes_write.sum, one launch each "
                          "(a wide stage = wide_windows gather window launches + the dense_tile launch); epoch average = "
                          "(4 wide + 2 narrow) / 6 for reddit"},
                  open(os.path.join(PROF, f"spmm_traffic_{wl}_P1.json"), "w"), indent=1)
    open(os.path.join(PROF, f"{tag}_summary.md"), "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
