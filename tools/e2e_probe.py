"""Where the pipelined run_host's time goes: kernel time (fused / band event sums, launches) of
the device path and of the pipelined e2e call, against their wall (event) times.

    python tools/e2e_probe.py heat3d [heat2d ...]
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

STEPS = {"heat3d": 100, "box3d27p": 100, "heat2d": 1000, "box2d49p": 200}


def timed(plan, fn, s):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    plan.set_profiling(True)
    e0.record(s)
    fn()
    e1.record(s)
    torch.cuda.synchronize()
    prof = plan.profile_read()
    plan.set_profiling(False)
    return e0.elapsed_time(e1), prof


for name in sys.argv[1:]:
    wk = wl.CONFIGS[name]
    plan = fs.Plan(wk.extents, wk.weights("seeded"), wk.radius, 0)
    u0 = wk.grid()
    st = STEPS[name]
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    s = torch.cuda.current_stream()
    h_in = torch.from_numpy(u0).pin_memory()
    h_out = torch.empty_like(h_in).pin_memory()
    plan.run(a, b, st, s)
    plan.run_host(h_in, h_out, st, s)
    torch.cuda.synchronize()
    for label, fn in (("device", lambda: plan.run(a, b, st, s)), ("e2e", lambda: plan.run_host(h_in, h_out, st, s))):
        for _ in range(2):
            ms, p = timed(plan, fn, s)
            info = plan.info()
            print(f"{name} {label}: wall {ms:.1f} ms  fused {p['fused_ms']:.1f} ms / {p['fused_launches']} launches "
                  f"({p['fused_ms'] / max(1, p['fused_launches']) * 1e3:.0f} us avg)  band {p['band_ms']:.1f} ms / "
                  f"{p['band_launches']}  K/Q {info['last_run_chunks']}/{info['last_run_depth']}", flush=True)
    plan.close()
    del a, b
    torch.cuda.empty_cache()
