"""A/B of programmatic dependent launch (FFTSTENCIL_PDL=0/1): device time of fftstencil_run with no
profiling events between the kernels, and the pipelined run_host, per workload.

    python tools/pdl_ab.py heat3d heat2d ...
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

STEPS = {"heat3d": 100, "box3d27p": 100, "heat2d": 1000, "box2d49p": 200, "star2d13p": 200}


def one(name, pdl, reps=5):
    os.environ["FFTSTENCIL_PDL"] = str(pdl)
    wk = wl.CONFIGS[name]
    plan = fs.Plan(wk.extents, wk.weights("seeded"), wk.radius, 0)
    u0 = wk.grid()
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    st = STEPS[name]
    s = torch.cuda.current_stream()
    for _ in range(2):
        plan.run(a, b, st, s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(reps):
        plan.run(a, b, st, s)
    e1.record(s)
    torch.cuda.synchronize()
    dev_ms = e0.elapsed_time(e1) / reps
    h_in = torch.from_numpy(u0).pin_memory()
    h_out = torch.empty_like(h_in).pin_memory()
    plan.run_host(h_in, h_out, st, s)
    torch.cuda.synchronize()
    e0.record(s)
    for _ in range(2):
        plan.run_host(h_in, h_out, st, s)
    e1.record(s)
    torch.cuda.synchronize()
    e2e_ms = e0.elapsed_time(e1) / 2
    ok = np.array_equal(h_out.numpy(), b.cpu().numpy())
    cells = float(np.prod(wk.extents)) * st
    print(f"{name} pdl={pdl} device {dev_ms:.2f} ms ({cells / dev_ms / 1e6:.1f} GSt/s)  e2e {e2e_ms:.2f} ms "
          f"({cells / e2e_ms / 1e6:.1f} GSt/s)  e2e==device {ok}", flush=True)
    plan.close()
    del a, b
    torch.cuda.empty_cache()


if __name__ == "__main__":
    for rep in range(2):
        for name in sys.argv[1:]:
            one(name, 0)
            one(name, 1)
