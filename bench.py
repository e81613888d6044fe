#!/usr/bin/env python
"""Benchmark of the B200-native FlashFFTStencil hot path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload heat2d] [--T 0] [--time-steps 1000]

One bench "step" = one fftstencil_run over the whole grid for `--time-steps` stencil time
steps (default: PAPER.md Table 3's 1000), i.e. one pass of every §8(a) row: ring copy,
floor(steps/T) fused FFT-tile passes + band passes, remainder pass.  The metric is
GStencils/s = cells x time steps / s / 1e9 (reading Q18), FP64.  Inputs are resident in
HBM for `value`; `e2e` goes through the C ABI's host-buffer entry point
(fftstencil_run_host) with the H2D/D2H copies inside the timed region.

--impl reference times the CPU oracle (oracle/, the plain direct stencil) on the host
cores on a bounded sample of the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import workloads as wl  # noqa: E402

FP64_PEAK_TFLOPS = 37.18   # measured DMMA.8x8x4 peak on this pool's B200 (profiles/r01_fp64_peak.txt)
# Measured FP64 instruction rates on this pool's B200 (tools/fp64_peak.cu, 8 independent chains
# per thread, 296 x 1024 threads; profiles/r01_s3_fp64_peak.txt), T instructions/s: DADD and
# DMUL issue at 64 per clock per SM, DFMA slightly slower.
FP64_RATES_TOPS = {"DADD": 18.51, "DMUL": 18.50, "DFMA": 17.05}
# FP64 instruction mix (DADD, DMUL, DFMA) of each default ALU kernel: static SASS counts of
# its TMA instantiation (cuobjdump -sass; the passes are straight-line code, so static =
# dynamic per thread and pair).  tests/test_bench.py re-counts them from the built objects.
ALU_KERNEL_MIX = {
    "kernel_fft2d_bf": (752, 168, 208),
    "kernel_fft3d_bf": (744, 92, 152),
    "kernel_fft1d_bf": (752, 292, 332),
}


def alu_peak_tops(mix) -> float:
    """Peak FP64 instruction rate for a kernel's mix: the time-weighted harmonic mean of the
    measured per-opcode rates (every DADD / DMUL / DFMA takes one FP64 pipe issue slot)."""
    n = sum(mix)
    return n / sum(k / FP64_RATES_TOPS[op] for k, op in zip(mix, ("DADD", "DMUL", "DFMA")))


FP64_ALU_PEAK_SOURCE = ("measured: tools/fp64_peak.cu per-opcode rates DADD 18.51 / DMUL 18.50 / DFMA 17.05 T "
                        "instructions/s (profiles/r01_s3_fp64_peak.txt), weighted by the kernel's SASS FP64 mix")
# Shared memory: 128 B per clock per SM (crossbar, /opt/skills/guides/B300_MICROARCH.md "LDS/STS"),
# 148 SMs at the 1.965 GHz max SM clock.
SMEM_PEAK_TBPS = 128 * 148 * 1.965e9 / 1e12


def smem_wavefronts_per_pair(info) -> float:
    """Designed shared-memory wavefronts (128 B each) per tile pair of the ALU kernels
    (DESIGN.md §5): every pass reads and writes the 64 KB complex pair (512 wavefronts each way)
    except where it is cropped, plus one read of S_T (512).  Twiddle-table loads and the TMA
    writes (async proxy) are not counted."""
    nd = info["ndim"]
    if nd == 2:       # P1..P4 read + write, P5 read, S_T
        return 9 * 512 + 512
    if nd == 3:       # P1, P2 full; P3 reads all, writes S planes; P4 on S planes; P5 on S^2 rows
        S = info["valid"][0]
        return 4 * 512 + 512 + 512 * S / 16 + 512 * S / 16 + 2 * 512 * S * S / 256 + 512
    return 13 * 512 + 512   # 1D: P1..P6 read + write, P7 read, S_T


FP64_PEAK_SOURCE = ("measured: tools/fp64_peak.cu DMMA m8n8k4 microbenchmark, 148 SMs x 64 FMA/clk x 1.965 GHz "
                    "(profiles/r01_fp64_peak.txt); MEASURED_PEAKS.json carries no FP64 figure")


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", default="heat2d", choices=sorted(wl.CONFIGS))
    ap.add_argument("--T", type=int, default=0, help="fused depth (0 = plan's automatic choice)")
    ap.add_argument("--time-steps", type=int, default=0, help="stencil time steps per bench step (0 = workload)")
    ap.add_argument("--weights", default="seeded", choices=["seeded", "classic"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--json-out", default="")
    return ap.parse_args()


def env_rank():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("LOCAL_RANK", "0")), int(os.environ.get("WORLD_SIZE", "1"))


class ClockSampler:
    """nvidia-smi sampling of SM clocks and throttle reasons during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *exc):
        self.lines = []
        if self.proc is not None:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()
                out = ""
            self.lines = [ln for ln in out.splitlines() if ln.strip()]

    def summary(self):
        sm, mx, reasons = [], [], set()
        for ln in getattr(self, "lines", []):
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
            for name, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(name)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


def kernel_name(info) -> str:
    """The fused kernel this plan launches (csrc/kernel_*.cu)."""
    nd, algo, L = info["ndim"], info["algo"], info["tile"][0]
    if nd == 1:
        if algo == "factored" and info.get("engine") == "alu":
            return "fft1d_bf_kernel (4096 = 64 x 64 four-step, 64 = 4 x 16 butterflies, FP64 ALU)"
        return "fft1d_ct_kernel (4096 = 64 x 64)" if algo == "factored" else "fft1d_kernel (PFA 8 x 7)"
    if nd == 2:
        if algo == "factored" and info.get("engine") == "alu":
            return "fft2d_bf_kernel (64 = 4 x 16 butterflies per axis, FP64 ALU)"
        return {"factored": "fft2d_ct_kernel (64 = 8 x 8 per axis)", "dense": f"fft2d_kernel<{L}>",
                "unfused": f"fft2d_kernel<{L}> forward / spec_mul / inverse"}[algo]
    if algo == "factored":
        return ("fft3d_bf_kernel (16 = 4 x 4 radix-4 FFT per line, FP64 ALU)" if info.get("engine") == "alu"
                else "fft3d_ct_kernel (16 = 8 x 2 per axis)")
    return "fft3d_kernel"


def load_traffic(info: dict, workload: str):
    """DRAM bytes per fused launch from the committed ncu --set full capture, if it matches."""
    path = os.path.join(ROOT, "profiles", "ncu_fused_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        e = d.get(workload)
        if (e and e.get("T") == info["T"] and e.get("tile") == info["tile"]
                and e.get("engine", "dmma") == info.get("engine", "dmma")):
            return float(e["dram_bytes_per_launch"])
    except Exception:
        pass
    return None


def gstencils(global_cells: int, time_steps: int, ms: float) -> float:
    """Whole-job GStencils/s (reading Q18): cells of the GLOBAL grid x stencil time steps / s.
    Under weak scaling the global grid already stacks every rank's slab, so no factor of the
    world size appears here (max-over-ranks time)."""
    return global_cells * time_steps / (ms / 1e3) / 1e9


def cpu_model() -> str:
    """The host CPU's model name (/proc/cpuinfo), reported beside the oracle's core count."""
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_oracle_sample(wk, w, budget_s: float = 12.0):
    """Time the oracle as it stands on the host cores on a bounded sample."""
    import oracle
    u = wk.grid()
    threads = oracle.max_threads()
    t0 = time.perf_counter()
    oracle.stencil_run(u, w, wk.radius, 1, nthreads=threads)
    t1 = time.perf_counter() - t0
    steps = 1
    if t1 < budget_s / 2:
        steps = int(max(1, min(64, budget_s / t1)))
        t0 = time.perf_counter()
        oracle.stencil_run(u, w, wk.radius, steps, nthreads=threads)
        t1 = time.perf_counter() - t0
    cells = int(np.prod(wk.extents))
    return {"value": cells * steps / t1 / 1e9, "unit": "GStencils/s", "cores": threads, "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"full {wk.name} grid {'x'.join(map(str, wk.extents))}, {steps} direct time step(s), "
                      f"{t1:.1f} s wall, OMP threads={threads}"}


def run_reference(args):
    rank, _, world = env_rank()
    if rank != 0:
        return 0
    import oracle
    wk = wl.CONFIGS[args.workload]
    w = wk.weights(args.weights)
    u = wk.grid()
    threads = oracle.max_threads()
    cells = int(np.prod(wk.extents))
    s_ref = 1   # direct time steps per bench step (bounded sample of the 1000-step run)
    for _ in range(args.warmup):
        oracle.stencil_run(u, w, wk.radius, s_ref, nthreads=threads)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.stencil_run(u, w, wk.radius, s_ref, nthreads=threads)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    value = cells * s_ref * args.steps / tot / 1e9
    line = {
        "impl": "reference", "metric": "GStencils/s FP64", "value": value, "unit": "GStencils/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{wk.name} {'x'.join(map(str, wk.extents))}"
                               + (" (BASELINE configs[1])" if args.workload in ("heat2d", "box2d9p") else ""),
                   "stencil": f"{wk.points}-point {wk.shape} r={wk.radius}, {args.weights} weights",
                   "time_steps_per_step": s_ref, "sample": "full grid, 1 direct time step per bench step"},
        "cpu_baseline": {"value": value, "unit": "GStencils/s", "cores": threads, "kind": "oracle",
                         "cpu_model": cpu_model(),
                         "sample": f"full grid, {s_ref} direct time step per bench step, {args.steps} timed"},
        "e2e": {"value": value, "unit": "GStencils/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs

    rank, local, world = env_rank()
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())

    wk = wl.CONFIGS[args.workload]
    w = wk.weights(args.weights)
    steps_per_run = args.time_steps or wk.bench_steps
    # weak scaling: each GPU keeps the N=1 workload's rows; the global grid stacks them
    # along axis 0 and the library decomposes it back into slabs (halo exchange by NCCL).
    gext = (wk.extents[0] * world,) + tuple(wk.extents[1:])
    cells = int(np.prod(gext))
    if world > 1:
        obj = [fs.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        plan = fs.Plan(gext, w, wk.radius, args.T or wk.T, nranks=world, rank=rank, nccl_id=obj[0])
        # this rank's slab of a seeded synthetic global grid (generated per slab)
        u0 = wl.grid(plan.extents, wk.cfg_id * 1000 + rank)
    else:
        plan = fs.Plan(gext, w, wk.radius, args.T or wk.T)
        u0 = wk.grid()
    info = plan.info()
    d_in = torch.from_numpy(u0).to(dev)
    d_out = torch.empty_like(d_in)
    stream = torch.cuda.current_stream(dev)

    def barrier():
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    for _ in range(max(args.warmup, 0)):
        plan.run(d_in, d_out, steps_per_run, stream)
    barrier()

    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    plan.set_profiling(True)
    with ClockSampler(dev.index) as clk:
        barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            plan.run(d_in, d_out, steps_per_run, stream)
        ev1.record(stream)
        barrier()
    prof = plan.profile_read()
    plan.set_profiling(False)
    launches_per_run = plan.info()["last_run_launches"]
    ms = ev0.elapsed_time(ev1)
    ms_t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms_max = float(ms_t.item())
    value = gstencils(cells, steps_per_run * args.steps, ms_max)

    # ---- roofline of the dominant kernel (the fused FFT-tile kernel) ----
    h = info["halo"]
    exact = max(0, min(info["row_end"], gext[0] - h) - max(info["row_begin"], h))   # this rank's exact rows
    for e in gext[1:]:
        exact *= max(0, e - 2 * h)
    passes = args.steps * -(-steps_per_run // info["T"])      # fused passes timed (1-3 launches each)
    fl = max(1, passes)
    fused_avg_s = prof["fused_ms"] / fl / 1e3
    alg_flops_launch = info["flops_per_cell_step"] * exact * info["T"]
    achieved = alg_flops_launch / fused_avg_s / 1e12
    traffic = load_traffic(info, args.workload)
    roofline = {"bound": "tensor", "achieved": achieved, "peak": FP64_PEAK_TFLOPS, "unit": "TFLOP/s",
                "frac": achieved / FP64_PEAK_TFLOPS, "traffic": traffic,
                "kernel": kernel_name(info),
                "dtype": "f64 (DMMA.8x8x4)", "peak_source": FP64_PEAK_SOURCE,
                "alg_flops_per_launch": alg_flops_launch,
                "flops_per_cell_step": info["flops_per_cell_step"],
                "mma_flops_per_launch": info["mma_flops_per_pass"],
                "mma_tflops": info["mma_flops_per_pass"] / fused_avg_s / 1e12,
                "fused_ms_avg": fused_avg_s * 1e3, "fused_share_of_step": prof["fused_ms"] / max(ms, 1e-9),
                "fused_launches": prof["fused_launches"], "passes": passes,
                "band_ms_avg": prof["band_ms"] / max(1, prof["band_launches"])}
    if info.get("engine") == "alu":
        # FP64 ALU engine: the binding unit is the FP64 pipe's issue rate (adds, multiplies and
        # FMAs each take one slot); peak = the measured DFMA rate / 2 (profiles/r01_fp64_peak.txt)
        ops = info["alu_ops_per_pass"] / fused_avg_s / 1e12
        mix = ALU_KERNEL_MIX[("kernel_fft1d_bf", "kernel_fft2d_bf", "kernel_fft3d_bf")[info["ndim"] - 1]]
        peak = alu_peak_tops(mix)
        roofline.update({"bound": "alu", "achieved": ops, "peak": peak, "unit": "Top/s",
                         "frac": ops / peak, "dtype": "f64 (DADD/DMUL/DFMA)", "fp64_mix": list(mix),
                         "peak_source": FP64_ALU_PEAK_SOURCE, "alu_ops_per_launch": info["alu_ops_per_pass"],
                         "alg_tflops": achieved})
        # the other unit the ALU kernels lean on (ncu: both below saturation)
        pairs = info["pair_end"] - info["pair_begin"]
        wf = smem_wavefronts_per_pair(info)
        smem_tbps = pairs * wf * 128 / fused_avg_s / 1e12
        roofline["smem"] = {"achieved": smem_tbps, "peak": SMEM_PEAK_TBPS, "unit": "TB/s",
                            "frac": smem_tbps / SMEM_PEAK_TBPS, "wavefronts_per_pair": wf,
                            "note": "designed LSU shared-memory traffic (no twiddle loads, no TMA writes) / "
                                    "fused-kernel time vs 128 B/clk/SM x 148 SMs x 1.965 GHz"}

    # ---- end to end through the host-buffer C-ABI entry point ----
    e2e = None
    if not args.no_e2e:
        h_in = torch.from_numpy(u0).pin_memory()
        h_out = torch.empty_like(h_in).pin_memory()
        plan.run_host(h_in, h_out, steps_per_run, stream)
        k_e = max(1, min(args.steps, 3))
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(k_e):
            plan.run_host(h_in, h_out, steps_per_run, stream)
        e1.record(stream)
        barrier()
        ems = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(ems, op=dist.ReduceOp.MAX)
        e_ms = float(ems.item())
        # whole job: every rank copies its slab in and its slab out each step
        e2e = {"value": gstencils(cells, steps_per_run * k_e, e_ms), "unit": "GStencils/s",
               "h2d_bytes_per_step": world * int(u0.nbytes), "d2h_bytes_per_step": world * int(u0.nbytes),
               "steps": k_e, "ms_per_step": e_ms / k_e, "api": "fftstencil_run_host (pinned host buffers)",
               "overlap": None if u0.ndim < 2 or world > 1 else ("copies overlapped with row-skewed passes: "
                           f"K={os.environ.get('FFTSTENCIL_E2E_PIPE', '6')} row chunks, "
                           f"Q={os.environ.get('FFTSTENCIL_E2E_DEPTH', '16')} skewed passes (DESIGN.md §6)")}
        if not np.isfinite(h_out.numpy()).all():
            raise RuntimeError("non-finite output")

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_oracle_sample(wk, w)

    if rank == 0:
        line = {
            "metric": "GStencils/s FP64", "value": value, "unit": "GStencils/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"{wk.name} {'x'.join(map(str, wk.extents))}"
                                   + (" (BASELINE configs[1])" if args.workload in ("heat2d", "box2d9p") else "")
                                   + ("" if world == 1 else f" per GPU; global {'x'.join(map(str, gext))}"),
                       "stencil": f"{wk.points}-point {wk.shape} r={wk.radius}, {args.weights} weights (seed 20250301)",
                       "grid": list(gext), "time_steps_per_step": steps_per_run, "T": info["T"],
                       "tile": info["tile"], "valid": info["valid"],
                       "parallelism": "single GPU" if world == 1 else
                       f"outer-axis decomposition over {world} GPUs, NCCL halo exchange of r*T rows per pass",
                       "l2": f"inputs {u0.nbytes / 1e6:.0f} MB > 126 MB L2 (no flush needed)"},
            "roofline": roofline,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(launches_per_run * args.steps),
            "clocks": clk.summary(),
        }
        s = json.dumps(line)
        print(s, flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(s + "\n")
    plan.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
