#!/usr/bin/env python
"""Summarise an ncu report (--set full) or a launch-list CSV into a small text file for profiles/.

    python tools/ncu_summary.py gpurun_out/r01_fft2d.ncu-rep > profiles/r01_fft2d_ncu.txt
    python tools/ncu_summary.py --launches gpurun_out/r01_launches.csv > profiles/r01_launches.txt
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

KEYS = [
    "Kernel Name", "gpu__time_duration.sum", "launch__grid_size", "launch__block_size",
    "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_shared_mem",
    "launch__occupancy_limit_registers", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_tensor_subpipe_dmma.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_bytes.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smsp__inst_executed.sum",
    "sm__cycles_elapsed.avg.per_second",
]


def summarise_report(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    for vals in rows[2:]:
        d = dict(zip(hdr, vals))
        u = dict(zip(hdr, units))
        print("=" * 100)
        for k in KEYS:
            if k in d:
                print(f"{k:80s} {d[k]} {u.get(k, '')}")
        stalls = []
        for h in hdr:
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    v = float(d[h].replace(",", ""))
                except ValueError:
                    continue
                stalls.append((v, h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
        print("warp stall reasons (warps per issue-active cycle):")
        for v, n in sorted(stalls, reverse=True):
            if v >= 0.02:
                print(f"   {n:30s} {v:.3f}")


def summarise_launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") != "gpu__time_duration.sum":
                continue
            agg[d["Kernel Name"]][0] += 1
            agg[d["Kernel Name"]][1] += float(d["Metric Value"].replace(",", ""))
    tot = sum(a[1] for a in agg.values()) or 1.0
    print(f"{'kernel':70s} {'launches':>8s} {'total ms':>10s} {'avg us':>10s} {'share':>7s}")
    for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{n[:70]:70s} {c:8d} {t / 1e6:10.3f} {t / c / 1e3:10.1f} {t / tot:7.3f}")


if __name__ == "__main__":
    if sys.argv[1] == "--launches":
        summarise_launches(sys.argv[2])
    else:
        summarise_report(sys.argv[1])
