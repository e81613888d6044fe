"""A/B of environment switches read at plan creation: device time of fftstencil_run (no profiling
events between kernels) and of the pipelined run_host, per workload and setting, two rounds.

    python tools/env_ab.py heat3d heat2d -- FFTSTENCIL_PDL=0 FFTSTENCIL_PDL=1
    python tools/env_ab.py heat3d -- FFTSTENCIL_BAND_STREAM=0 FFTSTENCIL_BAND_STREAM=1,FFTSTENCIL_E2E_BAND_SMS=8
(a setting is a comma-separated list of NAME=VALUE; "-" is the empty setting)
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

STEPS = {"heat3d": 100, "box3d27p": 100, "heat2d": 1000, "box2d49p": 200, "star2d13p": 200, "box2d9p": 1000}


def one(name, setting, reps=5):
    kv = [x.split("=", 1) for x in setting.split(",") if "=" in x]
    old = {k: os.environ.get(k) for k, _ in kv}
    os.environ.update({k: v for k, v in kv})
    try:
        wk = wl.CONFIGS[name]
        plan = fs.Plan(wk.extents, wk.weights("seeded"), wk.radius, 0)
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
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
    print(f"{name} [{setting}] device {dev_ms:.2f} ms ({cells / dev_ms / 1e6:.1f} GSt/s)  e2e {e2e_ms:.2f} ms "
          f"({cells / e2e_ms / 1e6:.1f} GSt/s)  e2e==device {ok}", flush=True)
    plan.close()
    del a, b
    torch.cuda.empty_cache()


if __name__ == "__main__":
    argv = sys.argv[1:]
    cut = argv.index("--") if "--" in argv else len(argv)
    names, settings = argv[:cut], (argv[cut + 1:] or ["-"])
    for rep in range(int(os.environ.get("ENV_AB_ROUNDS", "2"))):
        for name in names:
            for st in settings:
                one(name, st)
