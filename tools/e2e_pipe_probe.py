"""Probe of the pipelined run_host (capi.cu run_host_pipelined) on Heat-2D 10240^2, 1000 steps:
wall time per call, and the fused / band kernel time the plan's profiling events saw, for the
device path, the pipelined path and the unpipelined run_host.  Diagnostic only (not a bench).

    python tools/e2e_pipe_probe.py [K Q ...]
"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

ext, steps = (10240, 10240), 1000
w = wl.seeded_weights("star", 2, 1)
p = fs.Plan(ext, w, 1, 0)
u0 = wl.grid(ext, 1)
h_in = torch.from_numpy(u0).pin_memory()
h_out = torch.empty(ext, dtype=torch.float64).pin_memory()
a = h_in.cuda()
b = torch.empty_like(a)


def measure(label, fn, reps=3):
    fn()
    torch.cuda.synchronize()
    p.set_profiling(True)
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) * 1e3 / reps
    pr = p.profile_read()
    p.set_profiling(False)
    print(f"{label:28s} wall {wall:7.2f} ms  fused {pr['fused_ms'] / reps:7.2f} ms in {pr['fused_launches'] // reps} "
          f"launches, band {pr['band_ms'] / reps:6.2f} ms in {pr['band_launches'] // reps}", flush=True)


measure("device run", lambda: p.run(a, b, steps))
args = sys.argv[1:] or ["8", "16"]
os.environ["FFTSTENCIL_E2E_PIPE"] = "0"
measure("run_host unpipelined", lambda: p.run_host(h_in, h_out, steps))
for i in range(0, len(args), 2):
    os.environ["FFTSTENCIL_E2E_PIPE"], os.environ["FFTSTENCIL_E2E_DEPTH"] = args[i], args[i + 1]
    measure(f"run_host K={args[i]} Q={args[i + 1]}", lambda: p.run_host(h_in, h_out, steps))
ref = b.cpu().numpy()
assert np.array_equal(h_out.numpy(), ref), "pipelined result differs from the device path"
print("bitwise equal to the device path")
