"""Summarise tools/r02_table4.sh's ncu reports as a PAPER.md Table 4-style table (L340-L356).

UGA  = uncoalesced global accesses: excessive / total global sectors of the SourceCounters rule
       (0 when ncu raises no uncoalesced-access finding).
BC/R = shared-memory store bank conflicts per store request (STS); loads listed beside it.
PU   = pipeline utilisation of the line engine: FP64 pipe for the ALU engine, DMMA sub-pipe for the
       tensor engine (the paper's PU is its FP64 tensor-core pipe).
usage: python tools/table4_summary.py gpurun_out/t4 bench_log.txt
"""
import csv
import io
import re
import subprocess
import sys
from pathlib import Path


def raw(rep):
    out = subprocess.run(["ncu", "-i", str(rep), "--page", "raw", "--csv", "--print-units", "base"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return {}
    hdr, vals = rows[0], rows[2]
    d = {}
    for k, v in zip(hdr, vals):
        try:
            d[k] = float(v.replace(",", ""))
        except ValueError:
            d[k] = v
    return d


def uga(rep):
    out = subprocess.run(["ncu", "-i", str(rep), "--page", "details", "--print-details", "all"],
                         capture_output=True, text=True).stdout
    out = " ".join(out.split())
    m = re.search(r"uncoalesced global accesses resulting in a total of \d+ excessive sectors \((\d+(?:\.\d+)?)% of the total", out)
    return float(m.group(1)) if m else 0.0, out


def main():
    d = Path(sys.argv[1])
    bench = {}
    if len(sys.argv) > 2:
        for line in Path(sys.argv[2]).read_text().splitlines():
            if line.startswith("BENCH "):
                p = line.split()
                bench[(p[1], p[2])] = (float(p[3]), p[4])
    print("| kernel | engine / staging | GSt/s | fused ms | UGA % | BC/R st | BC/R ld | PU (FP64 pipe %) | PU (DMMA %) | LSU ld sect/req | LSU st sect/req | TMA load sectors |")
    print("|---|---|---|---|---|---|---|---|---|---|---|---|")
    for rep in sorted(d.glob("*.ncu-rep")):
        tag, w = rep.stem.split("_", 2)[:2], rep.stem.split("_", 2)[2]
        tag = "_".join(tag)
        m = raw(rep)
        if not m:
            continue
        g = lambda k: m.get(k, 0.0) if isinstance(m.get(k, 0.0), float) else 0.0
        st_req, ld_req = g("sm__sass_inst_executed_op_shared_st.sum"), g("sm__sass_inst_executed_op_shared_ld.sum")
        bcst = g("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum") / st_req if st_req else 0.0
        bcld = g("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum") / ld_req if ld_req else 0.0
        lr = g("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum") + g("l1tex__t_requests_pipe_lsu_mem_global_op_ldgsts_cache_access.sum")
        ls = g("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum") + g("l1tex__t_sectors_pipe_lsu_mem_global_op_ldgsts_cache_access.sum")
        sr, ss = g("l1tex__t_requests_pipe_lsu_mem_global_op_st.sum"), g("l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum")
        u, _ = uga(rep)
        b = bench.get((tag, w), (float("nan"), ""))
        print(f"| {m.get('Kernel Name', '?').split('(')[0].split('<')[0]} {w} | {tag} | {b[0]:.1f} | "
              f"{g('gpu__time_duration.sum') / 1e6:.3f} | {u:.1f} | {bcst:.2f} | {bcld:.2f} | "
              f"{g('sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | "
              f"{g('sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | "
              f"{ls / lr if lr else 0:.2f} | {ss / sr if sr else 0:.2f} | {g('l1tex__m_xbar2l1tex_read_sectors_mem_global_op_tma_ld.sum'):.3g} |")


if __name__ == "__main__":
    main()
