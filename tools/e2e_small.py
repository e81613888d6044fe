"""Small pipelined run_host calls (2D and 3D) compared bitwise with fftstencil_run, for
compute-sanitizer runs of the pipelined schedule."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

os.environ.setdefault("FFTSTENCIL_E2E_PIPE", "4")
os.environ.setdefault("FFTSTENCIL_E2E_DEPTH", "3")
for ext, shape, r, T, steps in [((800, 150), "box", 1, 4, 31), ((200, 30, 33), "star", 1, 2, 9)]:
    w = wl.seeded_weights(shape, len(ext), r)
    u0 = wl.grid(ext, 2)
    p = fs.Plan(ext, w, r, T)
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    p.run(a, b, steps)
    torch.cuda.synchronize()
    out = np.empty_like(u0)
    p.run_host(u0, out, steps)
    assert np.array_equal(out, b.cpu().numpy()), ext
    print(ext, "pipelined run_host bitwise equal, launches", p.info()["last_run_launches"])
