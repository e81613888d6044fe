"""Small runs of every kernel for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

torch.cuda.set_device(0)
F, D, C = "FFTSTENCIL_ALGO", "FFTSTENCIL_ENGINE", "FFTSTENCIL_MAX_CTAS"
cases = [((150, 140), "box", 1, 4, 9, {}), ((150, 140), "box", 1, 4, 9, {F: "dense"}),
         ((150, 140), "box", 1, 4, 9, {F: "factored", D: "dmma"}),
         ((130, 98), "star", 2, 3, 7, {"FFTSTENCIL_TMA": "0"}),
         ((40, 36, 34), "box", 1, 2, 5, {}), ((40, 36, 34), "box", 1, 2, 5, {F: "dense"}),
         ((40, 36, 34), "box", 1, 2, 5, {F: "factored", D: "dmma"}),
         ((33, 35, 37), "star", 1, 2, 3, {"FFTSTENCIL_TMA": "0"}), ((900,), "star", 1, 8, 19, {}),
         ((16384,), "star", 1, 1024, 1030, {F: "factored"}),                      # 1D ALU, TMA rows
         ((9000,), "star", 3, 352, 400, {F: "factored"}),                         # 1D ALU, cp.async
         ((9000,), "star", 3, 352, 400, {F: "factored", D: "dmma"}),
         # steady state of the persistent ALU kernels: one CTA, each group walks 5-20 pairs
         # through the TMA refill / mbarrier-parity loop (and the cp.async loop)
         ((300, 290), "box", 1, 8, 19, {C: "1"}), ((300, 290), "box", 1, 8, 19, {C: "1", "FFTSTENCIL_TMA": "0"}),
         ((60, 50, 45), "star", 1, 2, 5, {C: "1"}), ((60, 50, 45), "star", 1, 2, 5, {C: "1", "FFTSTENCIL_TMA": "0"}),
         ((65536,), "star", 2, 512, 1100, {C: "1", F: "factored"}),
         ((90001,), "star", 1, 300, 650, {C: "1", F: "factored"})]
for ext, shape, r, T, steps, env in cases:
    for k, v in env.items():
        os.environ[k] = v
    w = wl.seeded_weights(shape, len(ext), r)
    u = torch.from_numpy(wl.grid(ext, 3)).cuda()
    p = fs.Plan(ext, w, r, T)
    o = torch.empty_like(u)
    p.run(u, o, steps)
    torch.cuda.synchronize()
    assert np.isfinite(o.cpu().numpy()).all()
    print("ok", ext, env, p.info()["algo"], p.info()["engine"])
    for k in env:
        del os.environ[k]
# loopback decomposition
ext = (300, 130)
w = wl.seeded_weights("box", 2, 1)
u = torch.from_numpy(wl.grid(ext, 4)).cuda()
plans = [fs.Plan(ext, w, 1, 4, nranks=2, rank=k, loopback=True) for k in range(2)]
ins = [u[pl.info()["row_begin"]:pl.info()["row_end"]].contiguous() for pl in plans]
outs = [torch.empty_like(t) for t in ins]
fs.run_group(plans, ins, outs, 9)
torch.cuda.synchronize()
print("ok loopback")
