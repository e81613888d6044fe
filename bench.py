#!/usr/bin/env python
"""Benchmark of the B200-native FlashFFTStencil hot path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload NAME] [--T 0] [--time-steps 0] [--no-per-config]

One bench "step" = one fftstencil_run over the whole grid for `--time-steps` stencil time
steps (default: the workload's, Table 3's 1000 in 1D/2D, 100 in 3D), i.e. one pass
of every §8(a) row: ring copy, floor(steps/T) fused FFT-tile passes + band passes,
remainder pass.  The metric is GStencils/s = cells x time steps / s / 1e9 (reading Q18),
FP64.  Inputs are resident in HBM for `value`; `e2e` goes through the C ABI's host-buffer
entry point (fftstencil_run_host) with the H2D/D2H copies inside the timed region.

Workloads: N = 1 defaults to the largest single-GPU BASELINE config, Heat-3D
1024^3 (configs[3]); every other BASELINE config is measured in the same run and reported
under "per_config" (configs[0] Heat-1D 4096; configs[1] Heat-2D / Box-2D9P 10240^2 with the
T sweep; configs[2] Star-2D13P / Box-2D49P; configs[3] Box-3D27P; configs[4]'s per-GPU weak
slabs on one GPU, the denominator of the weak-scaling efficiency).  N > 1 defaults to
configs[4]'s weak slab Heat-3D (256 x 1024^2 per GPU, 2048 x 1024^2 at 8 GPUs).  Without
torchrun, `--gpus N > 1` re-launches itself under torch.distributed.run (one rank per GPU).

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


def _hbm_peak():
    """MEASURED_PEAKS.json hbm_gbs (driver-written copy bandwidth), else the profiling guide's
    fallback 6650 GB/s."""
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"])
    except Exception:
        return 6650.0


HBM_PEAK_GBS = _hbm_peak()


def alu_kernel_key(info) -> str:
    return ("kernel_fft1d_bf", "kernel_fft2d_bf", "kernel_fft3d_bf")[info["ndim"] - 1]


FP64_PEAK_SOURCE = ("measured: tools/fp64_peak.cu DMMA m8n8k4 microbenchmark, 148 SMs x 64 FMA/clk x 1.965 GHz "
                    "(profiles/r01_fp64_peak.txt); MEASURED_PEAKS.json carries no FP64 figure")


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", default="", choices=[""] + sorted(wl.CONFIGS),
                    help="default: heat3d at N = 1, heat3d_weak (configs[4]) at N > 1")
    ap.add_argument("--T", type=int, default=0, help="fused depth (0 = plan's automatic choice)")
    ap.add_argument("--time-steps", type=int, default=0, help="stencil time steps per bench step (0 = workload)")
    ap.add_argument("--weights", default="seeded", choices=["seeded", "classic"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-per-config", action="store_true", help="skip the other BASELINE configs (N = 1)")
    ap.add_argument("--json-out", default="")
    ap.add_argument("--transport", default="peer", choices=["peer", "nccl"],
                    help="N > 1 halo exchange: CUDA-IPC peer pushes + stream-memory signals (default) or NCCL send/recv")
    return ap.parse_args(argv)


def default_workload(world: int) -> str:
    """N = 1: the largest single-GPU BASELINE config (Heat-3D 1024^3, configs[3]); N > 1:
    configs[4]'s weak-scaled Heat-3D slab (256 x 1024^2 per GPU)."""
    return "heat3d" if world == 1 else "heat3d_weak"


# The other BASELINE configs measured beside the headline line at N = 1 (name, T, time steps
# per run; T = 0 is the plan's automatic choice).  configs[1]'s T sweep runs 240 time steps
# (a multiple of every swept T) per run.
PER_CONFIG = [
    ("heat1d", 8, 64, "configs[0]"),
    ("heat2d", 0, 1000, "configs[1]"),
    ("box2d9p", 0, 1000, "configs[1]"),
    *[(n, t, 240, "configs[1] T sweep") for n in ("heat2d", "box2d9p") for t in (1, 2, 4, 8, 12, 16)],
    ("star2d13p", 0, 1000, "configs[2]"),
    ("box2d49p", 0, 1000, "configs[2]"),
    ("heat3d", 0, 100, "configs[3]"),
    ("box3d27p", 0, 100, "configs[3]"),
    ("box2d9p_weak", 0, 1000, "configs[4] per-GPU slab, 1 GPU"),
    ("heat3d_weak", 0, 100, "configs[4] per-GPU slab, 1 GPU"),
    ("heat1d_512m", 0, 1000, "PAPER.md Table 3 L332 size (context)"),
]


def relaunch_under_torchrun(args_argv, n: int) -> int:
    """`--gpus N > 1` without a torch.distributed environment: run this script under
    torch.distributed.run with one rank per GPU (rendezvous on 127.0.0.1)."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *args_argv]
    return subprocess.call(cmd)


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
        if self.index < 0:   # sampling disabled
            return self
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


REF_SAMPLE_CELLS = 1 << 26   # ~67 M cells per direct step: a few seconds on the host cores


def cpu_oracle_sample(wk, w, budget_s: float = 12.0, u=None):
    """Time the oracle as it stands on the host cores on a bounded sample: the first outer rows
    of the workload grid (at most ~2^26 cells, the whole grid when smaller), as many direct
    time steps as fit in about `budget_s` seconds."""
    import oracle
    u = wk.grid() if u is None else u
    if u.ndim > 1 and u.size > REF_SAMPLE_CELLS:
        rows = max(2 * wk.radius + 2, REF_SAMPLE_CELLS // int(np.prod(u.shape[1:])))
        u = np.ascontiguousarray(u[:rows])
    threads = oracle.max_threads()
    t0 = time.perf_counter()
    oracle.stencil_run(u, w, wk.radius, 1, nthreads=threads)
    t1 = time.perf_counter() - t0
    steps = 1
    if t1 < budget_s / 2:
        steps = int(max(1, min(100000, budget_s / max(t1, 1e-6))))
        t0 = time.perf_counter()
        oracle.stencil_run(u, w, wk.radius, steps, nthreads=threads)
        t1 = time.perf_counter() - t0
    cells = int(u.size)
    whole = tuple(u.shape) == tuple(wk.extents)
    return {"value": cells * steps / t1 / 1e9, "unit": "GStencils/s", "cores": threads, "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"{'full' if whole else 'first outer rows of the'} {wk.name} grid: "
                      f"{'x'.join(map(str, u.shape))} cells, {steps} direct time step(s), "
                      f"{t1:.1f} s wall, OMP threads={threads}"}


def run_reference(args):
    """The oracle as it stands, timed on the host cores: each bench step is ONE direct time
    step over a bounded sample of the workload grid (its first outer rows, at most ~2^26 cells;
    the whole grid when smaller).  Rank 0 only; other ranks exit without work."""
    rank, _, world = env_rank()
    if rank != 0:
        return 0
    import oracle
    name = args.workload or default_workload(1)
    wk = wl.CONFIGS[name]
    w = wk.weights(args.weights)
    row = int(np.prod(wk.extents[1:])) if len(wk.extents) > 1 else 1
    rows = wk.extents[0] if len(wk.extents) == 1 else min(wk.extents[0],
                                                          max(2 * wk.radius + 2, REF_SAMPLE_CELLS // row))
    sample_ext = (rows,) + tuple(wk.extents[1:]) if len(wk.extents) > 1 else tuple(wk.extents)
    u = wk.grid(sample_ext)
    threads = oracle.max_threads()
    cells = int(np.prod(sample_ext))
    s_ref = 1   # direct time steps per bench step
    for _ in range(args.warmup):
        oracle.stencil_run(u, w, wk.radius, s_ref, nthreads=threads)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.stencil_run(u, w, wk.radius, s_ref, nthreads=threads)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    value = cells * s_ref * args.steps / tot / 1e9
    sample = (f"{'x'.join(map(str, sample_ext))} cells ({'whole grid' if rows == wk.extents[0] else 'first outer rows'}"
              f" of {'x'.join(map(str, wk.extents))}), {s_ref} direct time step per bench step, {args.steps} timed")
    line = {
        "impl": "reference", "metric": "GStencils/s FP64", "value": value, "unit": "GStencils/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{wk.name} {'x'.join(map(str, wk.extents))}"
                               + (" (BASELINE configs[3])" if not args.workload else ""),
                   "stencil": f"{wk.points}-point {wk.shape} r={wk.radius}, {args.weights} weights",
                   "time_steps_per_step": s_ref, "sample": sample},
        "cpu_baseline": {"value": value, "unit": "GStencils/s", "cores": threads, "kind": "oracle",
                         "cpu_model": cpu_model(), "sample": sample},
        "e2e": {"value": value, "unit": "GStencils/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def roofline_of(info, prof, passes, exact_cells, workload):
    """Roofline object of the dominant (fused FFT-tile) kernel: algorithmic work per launch over
    its average CUDA-event launch time, measured by the library on the launching stream."""
    fl = max(1, passes)
    fused_avg_s = prof["fused_ms"] / fl / 1e3
    alg_flops_launch = info["flops_per_cell_step"] * exact_cells * info["T"]
    achieved = alg_flops_launch / fused_avg_s / 1e12
    roof = {"bound": "tensor", "achieved": achieved, "peak": FP64_PEAK_TFLOPS, "unit": "TFLOP/s",
            "frac": achieved / FP64_PEAK_TFLOPS, "traffic": load_traffic(info, workload),
            "kernel": kernel_name(info), "dtype": "f64 (DMMA.8x8x4)", "peak_source": FP64_PEAK_SOURCE,
            "alg_flops_per_launch": alg_flops_launch, "flops_per_cell_step": info["flops_per_cell_step"],
            "mma_flops_per_launch": info["mma_flops_per_pass"],
            "mma_tflops": info["mma_flops_per_pass"] / fused_avg_s / 1e12,
            "fused_ms_avg": fused_avg_s * 1e3, "fused_launches": prof["fused_launches"], "passes": passes,
            "band_ms_avg": prof["band_ms"] / max(1, prof["band_launches"])}
    if info.get("engine") == "alu":
        # FP64 ALU engine: the binding unit is the FP64 pipe's issue rate (adds, multiplies and
        # FMAs each take one slot), peak = the measured per-opcode rates weighted by the kernel's mix
        ops = info["alu_ops_per_pass"] / fused_avg_s / 1e12
        mix = ALU_KERNEL_MIX[alu_kernel_key(info)]
        peak = alu_peak_tops(mix)
        roof.update({"bound": "alu", "achieved": ops, "peak": peak, "unit": "Top/s", "frac": ops / peak,
                     "dtype": "f64 (DADD/DMUL/DFMA)", "fp64_mix": list(mix), "peak_source": FP64_ALU_PEAK_SOURCE,
                     "alu_ops_per_launch": info["alu_ops_per_pass"], "alg_tflops": achieved})
        pairs = info["pair_end"] - info["pair_begin"]
        wf = smem_wavefronts_per_pair(info)
        smem_tbps = pairs * wf * 128 / fused_avg_s / 1e12
        roof["smem"] = {"achieved": smem_tbps, "peak": SMEM_PEAK_TBPS, "unit": "TB/s",
                        "frac": smem_tbps / SMEM_PEAK_TBPS, "wavefronts_per_pair": wf,
                        "note": "designed LSU shared-memory traffic (no twiddle loads, no TMA writes) / "
                                "fused-kernel time vs 128 B/clk/SM x 148 SMs x 1.965 GHz"}
    # HBM: the algorithmic traffic of one pass (read + write every cell once, 16 B/cell)
    cells = 1
    for e in info["extents"]:
        cells *= e
    hbm = 16.0 * cells / (prof["fused_ms"] / fl / 1e3) / 1e9
    roof["hbm"] = {"achieved": hbm, "peak": HBM_PEAK_GBS, "unit": "GB/s", "frac": hbm / HBM_PEAK_GBS,
                   "note": "16 B per grid cell per fused pass (read + write) / fused-kernel time, "
                           "vs MEASURED_PEAKS.json hbm_gbs"}
    return roof


def nccl_summary(path):
    """A few facts from rank 0's NCCL_DEBUG=INFO log (communicator setup of the halo exchange)."""
    try:
        txt = open(path, errors="replace").read()
    except OSError:
        return {"log": path, "found": False}
    return {"log": os.path.relpath(path, ROOT), "found": True, "init_complete": txt.count("Init COMPLETE"),
            "nvls": "NVLS" in txt, "p2p_or_nvlink": ("P2P" in txt) or ("NVL" in txt),
            "lines": txt.count("\n")}


def exact_cells_of(info, gext):
    h = info["halo"]
    exact = max(0, min(info["row_end"], gext[0] - h) - max(info["row_begin"], h))   # this rank's exact rows
    for e in gext[1:]:
        exact *= max(0, e - 2 * h)
    return exact


TRANSPORT_NOTE = []   # set when the peer transport had to fall back to NCCL (bench line config)


def peer_plan(fs, dist, world, rank, gext, w, radius, T):
    """A connected peer-transport plan, or None on EVERY rank if any rank failed (creation, handle
    export or mapping a neighbour's memory, e.g. devices without peer access): the group then
    falls back to NCCL together.  Each step is followed by an all-gather, so no rank is left
    waiting in a collective the others skipped."""
    def agree(err):
        errs = [None] * world
        dist.all_gather_object(errs, err)
        return [e for e in errs if e]

    plan, handle, err = None, None, ""
    try:
        plan = fs.Plan(gext, w, radius, T, nranks=world, rank=rank, transport="peer")
        handle = plan.peer_handle()
    except Exception as e:   # noqa: BLE001 -- reported in the line
        err = f"rank {rank}: {e}"
    handles = [None] * world
    dist.all_gather_object(handles, handle)
    errs = agree(err)
    if not errs:
        try:
            plan.peer_connect(handles[rank - 1] if rank > 0 else None, handles[rank + 1] if rank < world - 1 else None)
        except Exception as e:   # noqa: BLE001
            err = f"rank {rank}: {e}"
        errs = agree(err)
    if errs:
        if plan is not None:
            plan.close()
        TRANSPORT_NOTE.append("peer transport unavailable, fell back to NCCL: " + errs[0])
        return None
    return plan


def max_over_ranks(torch, dist, dev, world, x: float) -> float:
    """Max of a per-rank float over the group (a CPU tensor on a gloo group, CUDA on NCCL)."""
    if world == 1:
        return x
    on_gpu = dist.get_backend() == "nccl"
    t = torch.tensor([x], dtype=torch.float64, device=dev if on_gpu else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def measure(fs, torch, dist, dev, world, rank, name, T, time_steps, steps, warmup, weights="seeded",
            clocks=False, e2e=False, keep_input=False, transport="peer"):
    """Time `steps` fftstencil_run calls of `time_steps` time steps each on workload `name`
    (weak scaling: each rank holds the workload's rows, the global grid stacks them)."""
    wk = wl.CONFIGS[name]
    w = wk.weights(weights)
    gext = (wk.extents[0] * world,) + tuple(wk.extents[1:])
    cells = int(np.prod(gext))
    plan = None
    if world > 1 and transport == "peer":
        plan = peer_plan(fs, dist, world, rank, gext, w, wk.radius, T)
        if plan is None:
            transport = "nccl"
    if plan is not None:
        u0 = wl.grid(plan.extents, wk.cfg_id * 1000 + rank)   # this rank's slab, seeded per slab
    elif world > 1:
        obj = [fs.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        plan = fs.Plan(gext, w, wk.radius, T, nranks=world, rank=rank, nccl_id=obj[0])
        u0 = wl.grid(plan.extents, wk.cfg_id * 1000 + rank)   # this rank's slab, seeded per slab
    else:
        plan = fs.Plan(gext, w, wk.radius, T)
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

    for _ in range(max(warmup, 0)):
        plan.run(d_in, d_out, time_steps, stream)
    barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    plan.set_profiling(True)
    with ClockSampler(dev.index if clocks else -1) as clk:
        barrier()
        ev0.record(stream)
        for _ in range(steps):
            plan.run(d_in, d_out, time_steps, stream)
        ev1.record(stream)
        barrier()
    prof = plan.profile_read()
    plan.set_profiling(False)
    launches = plan.info()["last_run_launches"]
    peer_fused = plan.info()["last_run_peer_fused"]
    ms = ev0.elapsed_time(ev1)
    ms_max = max_over_ranks(torch, dist, dev, world, ms)
    passes = steps * -(-time_steps // info["T"])
    res = {"workload": name, "value": gstencils(cells, time_steps * steps, ms_max), "unit": "GStencils/s",
           "ms_per_step": ms_max / steps, "steps": steps, "time_steps_per_step": time_steps,
           "T": info["T"], "tile": info["tile"], "valid": info["valid"], "grid": list(gext),
           "gpu_launches_per_step": int(launches), "peer_fused": bool(peer_fused),
           "roofline": roofline_of(info, prof, passes, exact_cells_of(info, gext), name),
           "fused_share_of_step": prof["fused_ms"] / max(ms, 1e-9)}
    res["roofline"]["fused_share_of_step"] = res["fused_share_of_step"]
    if clocks:
        res["clocks"] = clk.summary()
    if e2e:
        h_in = torch.from_numpy(u0).pin_memory()
        h_out = torch.empty_like(h_in).pin_memory()
        plan.run_host(h_in, h_out, time_steps, stream)
        k_e = max(1, min(steps, 3))
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(k_e):
            plan.run_host(h_in, h_out, time_steps, stream)
        e1.record(stream)
        barrier()
        e_ms = max_over_ranks(torch, dist, dev, world, e0.elapsed_time(e1))
        pinfo = plan.info()
        piped = pinfo["last_run_pipelined"]
        res["e2e"] = {"value": gstencils(cells, time_steps * k_e, e_ms), "unit": "GStencils/s",
                      "h2d_bytes_per_step": world * int(u0.nbytes), "d2h_bytes_per_step": world * int(u0.nbytes),
                      "steps": k_e, "ms_per_step": e_ms / k_e, "api": "fftstencil_run_host (pinned host buffers)",
                      "pipelined": piped,
                      "overlap": ("copies overlapped with row-skewed passes: "
                                  f"K={pinfo['last_run_chunks']} row chunks, "
                                  f"Q={pinfo['last_run_depth']} skewed passes (DESIGN.md §6)")
                      if piped else "none: copy-run-copy (the plan does not take the pipelined schedule)"}
        if not np.isfinite(h_out.numpy()).all():
            raise RuntimeError("non-finite output")
    if world > 1:
        barrier()   # no rank frees buffers a neighbour still has mapped (peer transport)
    plan.close()
    if keep_input:
        res["_u0"] = u0
    del d_in, d_out
    torch.cuda.empty_cache()
    return res


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    args = parse(argv)
    if args.impl == "reference":
        return run_reference(args)
    rank, local, world = env_rank()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch_under_torchrun(argv, args.gpus)
    if world != args.gpus and "WORLD_SIZE" in os.environ:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}: launch one rank per GPU")

    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs

    nccl_log = None
    shared = os.environ.get("FFTSTENCIL_BENCH_SHARE_GPU") == "1"
    if world > 1 and args.transport == "nccl":
        # the library's own communicator (ncclCommInitRank in fftstencil_plan_create_dist) logs
        # its setup -- transport, NVLS, channels -- to a file, so stdout keeps the one JSON line
        nccl_log = os.path.join(ROOT, "gpurun_out", f"nccl_rank{rank}.log")
        os.makedirs(os.path.dirname(nccl_log), exist_ok=True)
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_FILE", nccl_log)
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    elif world > 1:
        # peer transport: the library moves the halos itself (CUDA IPC); the harness only needs
        # a barrier and a max over ranks, over gloo.  FFTSTENCIL_BENCH_SHARE_GPU=1 (harness test
        # on a one-GPU box) puts every rank on device 0 -- not a scaling measurement.
        torch.cuda.set_device(local % torch.cuda.device_count() if shared else local)
        dist.init_process_group("gloo")
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    name = args.workload or default_workload(world)
    wk = wl.CONFIGS[name]
    time_steps = args.time_steps or wk.bench_steps
    main_res = measure(fs, torch, dist, dev, world, rank, name, args.T or wk.T, time_steps, args.steps,
                       args.warmup, args.weights, clocks=True, e2e=not args.no_e2e,
                       keep_input=world == 1 and not args.no_cpu_baseline, transport=args.transport)

    u_main = main_res.pop("_u0", None)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_oracle_sample(wk, wk.weights(args.weights), u=u_main)
    del u_main

    per_config = None
    if world == 1 and not args.no_per_config:
        per_config = []
        for pname, pT, pts, label in PER_CONFIG:
            if pname == name and pT == 0 and not args.T:
                continue   # the headline line itself
            pk = wl.CONFIGS[pname]
            small = int(np.prod(pk.extents)) < (1 << 20)
            want_cpu = not args.no_cpu_baseline and (pT == 0 or pname == "heat1d")
            r = measure(fs, torch, dist, dev, 1, 0, pname, pT or pk.T, pts, 200 if small else 2,
                        20 if small else 1, args.weights, keep_input=want_cpu)
            r["baseline_config"] = label
            r["stencil"] = f"{pk.points}-point {pk.shape} r={pk.radius}"
            u_host = r.pop("_u0", None)
            if want_cpu:
                r["cpu_baseline"] = cpu_oracle_sample(pk, pk.weights(args.weights), budget_s=3.0, u=u_host)
            del u_host
            per_config.append(r)

    if rank == 0:
        line = {
            "metric": "GStencils/s FP64", "value": main_res["value"], "unit": "GStencils/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": main_res["ms_per_step"],
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"{wk.name} {'x'.join(map(str, wk.extents))}"
                                   + {"heat3d": " (BASELINE configs[3], largest single-GPU config)",
                                      "heat3d_weak": " (BASELINE configs[4] weak slab)",
                                      "box2d9p_weak": " (BASELINE configs[4] weak slab)"}.get(name, "")
                                   + ("" if world == 1 else f" per GPU; global {'x'.join(map(str, main_res['grid']))}"),
                       "stencil": f"{wk.points}-point {wk.shape} r={wk.radius}, {args.weights} weights (seed 20250301)",
                       "grid": main_res["grid"], "time_steps_per_step": time_steps, "T": main_res["T"],
                       "tile": main_res["tile"], "valid": main_res["valid"],
                       "parallelism": "single GPU" if world == 1 else
                       f"outer-axis decomposition over {world} GPUs, r*T halo rows per pass "
                       + ("pushed into the neighbours' buffers (CUDA IPC peer copies, stream-memory signal/wait)"
                          if args.transport == "peer" and not TRANSPORT_NOTE else "by NCCL send/recv"),
                       "l2": f"inputs {int(np.prod(wk.extents)) * 8 / 1e6:.0f} MB per GPU > 126 MB L2 (no flush needed)"},
            "roofline": main_res["roofline"],
            "cpu_baseline": cpu,
            "e2e": main_res.get("e2e"),
            "gpu_launches": int(main_res["gpu_launches_per_step"] * args.steps),
            "clocks": main_res["clocks"],
            "per_config": per_config,
        }
        if nccl_log:
            line["config"]["nccl"] = nccl_summary(nccl_log)
        if world > 1:
            line["config"]["transport"] = (("peer: halo rows stored into the neighbours by the edge tiles' and band's kernels"
                                            if main_res.get("peer_fused") else "peer: halo rows copied after each pass")
                                           if args.transport == "peer" and not TRANSPORT_NOTE else "nccl")
            if TRANSPORT_NOTE:
                line["config"]["transport_note"] = TRANSPORT_NOTE[0]
        if world > 1 and shared:
            line["shared_gpu"] = "every rank on device 0 (FFTSTENCIL_BENCH_SHARE_GPU=1): a harness test, not a scaling number"
        s = json.dumps(line)
        print(s, flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(s + "\n")
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
